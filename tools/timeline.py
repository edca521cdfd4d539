#!/usr/bin/env python3
"""Launch timeline of one concurrent step (timing mode 3) on the headline grid: per-stream busy
time, idle gaps, and how much of the step two or more streams overlap.  Run on the GPU box:
    python tools/timeline.py [--config 3] [--chunk-pairs 64] [--chunk-tiles 32] [--csv out.csv]
"""
import argparse
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import synthgrid  # noqa: E402
from paper_conf_icpp_blattnerkcsbz14_b200 import PciamGrid  # noqa: E402

NAMES = ["K1", "K2", "K3", "K4", "K5", "K6"]
STREAMS = ["forward", "pairs", "ccf"]


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", type=int, default=3)
    ap.add_argument("--chunk-pairs", type=int, default=0)
    ap.add_argument("--chunk-tiles", type=int, default=0)
    ap.add_argument("--csv", default="")
    a = ap.parse_args()
    g = synthgrid.make_config(a.config)
    with PciamGrid(g.n, g.m, g.H, g.W, chunk_pairs=a.chunk_pairs, chunk_tiles=a.chunk_tiles) as pg:
        pg.load_grid(g.tiles)
        for _ in range(2):
            pg.compute_translations()
        pg.set_timing(3)
        pg.compute_translations()
        tl = pg.timeline()
    k, s, t0, t1 = tl["kernel"], tl["stream"], tl["start_ms"], tl["end_ms"]
    end = float(t1.max())
    print(f"step {end:.2f} ms, {len(k)} launches")
    for si, name in enumerate(STREAMS):
        m = s == si
        busy = float((t1[m] - t0[m]).sum())
        first, last = float(t0[m].min()), float(t1[m].max())
        print(f"  {name:8s} busy {busy:7.2f} ms  span [{first:6.2f}, {last:6.2f}]  "
              f"idle inside span {last - first - busy:6.2f} ms")
    for ki, name in enumerate(NAMES):
        m = k == ki
        if m.any():
            print(f"  {name}: {int(m.sum()):4d} launches, {float((t1[m] - t0[m]).sum()):7.2f} ms "
                  f"in flight (concurrent, so longer than alone)")
    # overlap: time covered by >= 1 / >= 2 / 3 streams (1 us grid)
    grid = np.zeros((3, int(end * 1000) + 1), bool)
    for ki, si, a0, a1 in zip(k, s, t0, t1):
        grid[si, int(a0 * 1000): int(a1 * 1000)] = True
    c = grid.sum(0)
    print(f"  time with >=1 stream busy {np.count_nonzero(c >= 1) / 1000:.2f} ms, >=2 "
          f"{np.count_nonzero(c >= 2) / 1000:.2f} ms, 3 {np.count_nonzero(c >= 3) / 1000:.2f} ms")
    if a.csv:
        with open(a.csv, "w") as f:
            f.write("kernel,stream,start_ms,end_ms\n")
            for row in zip(k, s, t0, t1):
                f.write(f"{NAMES[row[0]]},{STREAMS[row[1]]},{row[2]:.4f},{row[3]:.4f}\n")


if __name__ == "__main__":
    main()
