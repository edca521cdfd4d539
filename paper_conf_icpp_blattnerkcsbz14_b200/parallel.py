"""Row-band multi-GPU partition of a PCIAM grid.

The paper runs one independent pipeline per GPU over a spatial decomposition of the
grid and leaves the partition boundary unspecified (reading C16);
P2P copies between cards are its future work (L1512-1517).  Here:

* rank k of R owns the tiles [k*nt/R, (k+1)*nt/R) (row-major, nt = n*m) and the pairs
  whose tile B it owns (Fig. 4 west/north pairs);
* its pairs also need the m tiles before its first tile (one tile row, the "halo"):
  their raw pixels are loaded with the band, their spectra are RECEIVED from rank k-1,
  which owns them and has just transformed them -- one point-to-point send/recv per band
  boundary (NCCL over NVLink through torch.distributed; gloo in the CPU tests);
* results are merged with one all_gather of each rank's owned entries.

If a band is shorter than a tile row the halo spans two ranks; the driver then falls
back to recomputing the halo's forward transforms locally (no data-path collective).
torch is plumbing here: process groups, the workspace tensor, the stream.
"""
from __future__ import annotations

from dataclasses import dataclass

import numpy as np


@dataclass(frozen=True)
class Band:
    rank: int
    world: int
    t_begin: int      # first owned tile
    t_end: int        # one past the last owned tile
    halo_begin: int   # first resident tile = max(0, t_begin - m)
    row_begin: int    # tile rows [row_begin, row_end) hold every resident tile
    row_end: int

    @property
    def owned(self) -> int:
        return self.t_end - self.t_begin


def band(rank: int, world: int, n: int, m: int) -> Band:
    nt = n * m
    if not (0 <= rank < world) or world < 1:
        raise ValueError("bad rank/world")
    b, e = rank * nt // world, (rank + 1) * nt // world
    halo = max(0, b - m)
    return Band(rank, world, b, e, halo, halo // m, (e - 1) // m + 1 if e > 0 else 0)


@dataclass(frozen=True)
class HaloPlan:
    """Tile ranges this rank sends to rank+1 / receives from rank-1 (None: nothing)."""
    send: tuple[int, int] | None   # (first tile, count)
    recv: tuple[int, int] | None


def exchange_feasible(world: int, n: int, m: int) -> bool:
    """Every halo lies inside the previous rank's band (all bands >= one tile row)."""
    return world > 1 and all(band(k, world, n, m).owned >= m for k in range(world - 1))


def halo_plan(rank: int, world: int, n: int, m: int) -> HaloPlan:
    bd = band(rank, world, n, m)
    recv = (bd.halo_begin, bd.t_begin - bd.halo_begin) if rank > 0 and bd.t_begin > 0 else None
    send = None
    if rank < world - 1:
        nxt = band(rank + 1, world, n, m)
        cnt = nxt.t_begin - nxt.halo_begin
        if cnt > 0:
            send = (nxt.halo_begin, cnt)
    if recv and recv[1] == 0:
        recv = None
    return HaloPlan(send, recv)


def exchange_halo(send_buf, recv_buf, rank: int, world: int, group=None) -> None:
    """Send `send_buf` to rank+1 and receive `recv_buf` from rank-1 (batched P2P).  NCCL moves
    device buffers GPU to GPU; under gloo (CPU tests, or the bench's --dist-backend gloo logic
    check) device buffers are staged through host memory."""
    import torch.distributed as dist
    if dist.get_backend(group) == "gloo" and any(b is not None and b.is_cuda
                                                 for b in (send_buf, recv_buf)):
        import torch
        torch.cuda.current_stream().synchronize()
        s_host = send_buf.cpu() if send_buf is not None else None
        r_host = torch.empty_like(recv_buf, device="cpu") if recv_buf is not None else None
        exchange_halo(s_host, r_host, rank, world, group)
        if recv_buf is not None:
            recv_buf.copy_(r_host)
        return
    ops = []
    if send_buf is not None and rank + 1 < world:
        ops.append(dist.P2POp(dist.isend, send_buf, rank + 1, group))
    if recv_buf is not None and rank > 0:
        ops.append(dist.P2POp(dist.irecv, recv_buf, rank - 1, group))
    if ops:
        for w in dist.batch_isend_irecv(ops):
            w.wait()


def gather_translations(west: np.ndarray, north: np.ndarray, bd: Band, group=None):
    """Merge every rank's owned entries into full [n, m] arrays on all ranks."""
    import torch.distributed as dist
    mine = (bd.t_begin, bd.t_end, west.reshape(-1)[bd.t_begin:bd.t_end].copy(),
            north.reshape(-1)[bd.t_begin:bd.t_end].copy())
    parts = [None] * bd.world
    dist.all_gather_object(parts, mine, group=group)
    w, n = west.copy().reshape(-1), north.copy().reshape(-1)
    for b, e, pw, pn in parts:
        w[b:e] = pw
        n[b:e] = pn
    return w.reshape(west.shape), n.reshape(north.shape)


class BandPciam:
    """One rank's share of a grid: a PciamGrid over its band plus the halo exchange.

    transport:
      "library"   -- the library's own NCCL send/recv (stitch_config.nccl_id; rank 0 makes the
                     id, torch.distributed broadcasts it): one call per step, the exchange on
                     the library's comm stream overlapped with the interior pairs;
      "torch"     -- the same exchange through torch.distributed (NCCL, or gloo staging through
                     host memory in the CPU tests) on a side stream, overlapped the same way:
                     forward(owned) -> [interior pairs || halo exchange] -> boundary pairs;
      "recompute" -- no exchange: the halo row's forward transforms are recomputed locally.
    The exchange needs every band but the last to hold >= one tile row (exchange_feasible);
    otherwise every transport falls back to "recompute"."""

    def __init__(self, n: int, m: int, H: int, W: int, rank: int, world: int, device: int = 0,
                 exchange: bool = True, group=None, transport: str | None = None, **kw):
        from . import PciamGrid, nccl_unique_id
        self.n, self.m, self.H, self.W = n, m, H, W
        self.rank, self.world, self.group = rank, world, group
        self.bd = band(rank, world, n, m)
        self.plan = halo_plan(rank, world, n, m)
        if transport is None:
            transport = "torch" if exchange else "recompute"
        if transport not in ("library", "torch", "recompute"):
            raise ValueError("transport must be library, torch or recompute")
        if not exchange_feasible(world, n, m):
            transport = "recompute"
        self.transport = transport
        self.use_exchange = transport != "recompute"
        if transport == "library":
            import torch.distributed as dist
            obj = [nccl_unique_id() if rank == 0 else None]
            dist.broadcast_object_list(obj, src=0, group=group)
            self.grid = PciamGrid(n, m, H, W, device=device, rank=rank, world_size=world,
                                  nccl_id=obj[0], **kw)
        else:
            self.grid = PciamGrid(n, m, H, W, device=device, tile_begin=self.bd.t_begin,
                                  tile_end=self.bd.t_end, **kw)
        assert (self.grid.tile_begin, self.grid.tile_end) == (self.bd.t_begin, self.bd.t_end)
        self.npairs = self.grid.npairs
        self._comm_stream = None

    def load_rows(self, rows, first_tile: int | None = None) -> None:
        """Tiles of rows [row_begin, row_end) ([rows, m, H, W], host or device)."""
        self.grid.load_tiles(rows, self.bd.row_begin * self.m if first_tile is None
                             else first_tile)

    def step_async(self) -> None:
        """Steps 2-7 for the band: forward the owned tiles; then the interior pairs while the
        halo row's spectra move from rank-1 (and this band's last row to rank+1); then the
        boundary pairs (tile A in the halo)."""
        if self.transport in ("recompute", "library"):
            self.grid.compute_translations_async()     # halo recomputed / exchanged inside
            return
        import torch
        g = self.grid
        g.forward_range_async(self.bd.t_begin, self.bd.owned)
        fwd_done = torch.cuda.Event()
        fwd_done.record(g.stream)
        g.pairs_async(1)                               # interior: no halo spectrum needed
        if self._comm_stream is None:
            self._comm_stream = torch.cuda.Stream(g.device)
        cs = self._comm_stream
        cs.wait_event(fwd_done)
        send = g.spectra_view(*self.plan.send) if self.plan.send else None
        recv = g.spectra_view(*self.plan.recv) if self.plan.recv else None
        with torch.cuda.stream(cs):                    # exchange beside the interior pairs
            exchange_halo(send, recv, self.rank, self.world, self.group)
        g.stream.wait_stream(cs)
        g.pairs_async(2)                               # boundary pairs after the halo landed

    def translations(self):
        return self.grid.get_translations()

    def close(self) -> None:
        self.grid.close()
