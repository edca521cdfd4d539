"""Streaming time series of grids (BASELINE.json configs[3]).

The paper's motivating experiment scans a plate 161 times, two channels per scan, each an
18x22 grid of 1392x1040 tiles -- 344 GB of raw data -- and its
system bounds memory with a fixed buffer pool, per-tile reference counts and a traversal
order, while a pipeline overlaps disk, PCIe, GPU and CPU.

On B200 one grid's whole working set (tiles 1.15 GB + phase spectra 1.15 GB + chunk
intermediates) fits HBM many times over, so the bounded pool becomes a fixed number of
grid *slots*: each slot is one library context (own workspace, own stream, own pinned
host staging buffer).  Grid g goes to slot g mod S: its host-side fill, H2D copy, the
forward/pair/CCF kernels and the D2H of its results run on that slot's stream while the
other slots' work proceeds, so PCIe transfers overlap GPU compute.  Device memory is
S x (one grid's workspace), independent of the series length.  Multi-GPU: whole grids
are dealt round-robin to the ranks (independent problems, no data-path collective).
"""
from __future__ import annotations

import os
from dataclasses import dataclass
from typing import Callable, Iterable

import numpy as np

from . import PciamGrid


@dataclass
class GridResult:
    index: int
    west: np.ndarray
    north: np.ndarray


class ResultStore:
    """Per-scan resumability of a time series: each finished
    grid's (west, north) records go to their own file `grid_<index>.npz` in `directory`,
    written to a temporary name and renamed into place, so a file present is a complete
    result and a run that stops (crash, preemption) loses at most the grids in flight.
    A restarted stream skips every index already stored."""

    PREFIX, SUFFIX = "grid_", ".npz"

    def __init__(self, directory: str):
        self.dir = directory
        os.makedirs(directory, exist_ok=True)

    def path(self, index: int) -> str:
        return os.path.join(self.dir, f"{self.PREFIX}{index:07d}{self.SUFFIX}")

    def done(self) -> set[int]:
        out = set()
        for f in os.listdir(self.dir):
            if f.startswith(self.PREFIX) and f.endswith(self.SUFFIX):
                try:
                    out.add(int(f[len(self.PREFIX):-len(self.SUFFIX)]))
                except ValueError:
                    pass
        return out

    def save(self, r: GridResult) -> None:
        tmp = os.path.join(self.dir, f".tmp_{r.index}_{os.getpid()}.npz")
        with open(tmp, "wb") as f:
            np.savez(f, west=r.west, north=r.north)
            f.flush()
            os.fsync(f.fileno())
        os.replace(tmp, self.path(r.index))

    def load(self, index: int) -> GridResult:
        with np.load(self.path(index)) as z:
            return GridResult(index, z["west"], z["north"])


def pending(indices: Iterable[int], store: ResultStore | None) -> list[int]:
    """The indices still to run (in order): all of them, or those the store lacks."""
    indices = list(indices)
    if store is None:
        return indices
    done = store.done()
    return [i for i in indices if i not in done]


class GridStream:
    """S slots of one context each; `run` streams grids through them."""

    def __init__(self, n: int, m: int, H: int, W: int, slots: int = 2, device: int = 0, **kw):
        import torch
        self.n, self.m, self.H, self.W = n, m, H, W
        self.slots = []
        for _ in range(slots):
            stream = torch.cuda.Stream(device)
            with torch.cuda.stream(stream):
                g = PciamGrid(n, m, H, W, device=device, **kw)
            host = torch.empty((n, m, H, W), dtype=torch.uint16, pin_memory=True)
            self.slots.append({"grid": g, "host": host, "pending": None})
        self.pairs_per_grid = self.slots[0]["grid"].npairs

    def run(self, indices: Iterable[int], fill: Callable[[int, np.ndarray], object],
            sink: Callable[[GridResult], None] | None = None,
            store: ResultStore | None = None) -> int:
        """For each grid index: fill(index, host_array) either writes its tiles into the
        slot's pinned buffer (returning None) or returns a pinned host tensor / array that
        already holds them; then H2D + steps 2-7 are enqueued on the slot's stream.
        Results are collected (saved to `store`, then passed to `sink`) when the slot comes
        round again; with a store, indices it already holds are skipped (resume).
        Returns the number of grids processed."""
        count = 0
        S = len(self.slots)
        self._store = store
        for k, idx in enumerate(pending(indices, store)):
            sl = self.slots[k % S]
            if sl["pending"] is not None:
                self._collect(sl, sink)
            src = fill(idx, sl["host"].numpy())
            sl["src"] = src                      # keep the source alive until collected
            # steps 1-7 on the slot's stream, the H2D pipelined per forward chunk
            sl["grid"].compute_from_host_async(sl["host"] if src is None else src, 0)
            sl["pending"] = idx
            count += 1
        for sl in self.slots:
            if sl["pending"] is not None:
                self._collect(sl, sink)
        return count

    def _collect(self, sl, sink):
        w, n = sl["grid"].get_translations()          # D2H of the results, synchronous
        r = GridResult(sl["pending"], w.copy(), n.copy())
        if getattr(self, "_store", None) is not None:
            self._store.save(r)
        if sink is not None:
            sink(r)
        sl["pending"] = None

    def close(self) -> None:
        for sl in self.slots:
            sl["grid"].close()
        self.slots = []

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()


def shard(indices: list[int], rank: int, world: int) -> list[int]:
    """Whole grids dealt round-robin to ranks (the time series shards without exchange)."""
    return indices[rank::world]
