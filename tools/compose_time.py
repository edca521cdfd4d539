#!/usr/bin/env python3
"""Time phase 3 (stitch_compose_overlay) on the 42x59 grid at its generator positions (B200)."""
import os
import sys
import time

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import synthgrid  # noqa: E402
from paper_conf_icpp_blattnerkcsbz14_b200 import compose_overlay  # noqa: E402

g = synthgrid.make_config(3)
tiles = torch.from_numpy(g.tiles.view(np.int16)).view(torch.uint16).cuda()
pos = g.origins - g.origins.min(axis=(0, 1))
canvas = compose_overlay(tiles, pos)
torch.cuda.synchronize()
ts = []
for _ in range(5):
    t0 = time.perf_counter()
    compose_overlay(tiles, pos, canvas)
    torch.cuda.synchronize()
    ts.append(time.perf_counter() - t0)
c = canvas.cpu().numpy()
print(f"{sys.argv[1] if len(sys.argv) > 1 else ''} compose {1e3 * min(ts):.2f} ms (min of 5), canvas "
      f"{c.shape}, checksum {int(c.astype(np.uint64).sum())}")
