#!/bin/bash
# compute-sanitizer passes over config 1 (3x3 grid of 256x192) and a 2x2 grid of 1392x1040
# (run on the GPU box).  Graph replay off so every launch is checked directly.
SMOKE='import __graft_entry__ as g; g.smoke()'
BIG='import numpy as np, torch, synthgrid; from paper_conf_icpp_blattnerkcsbz14_b200 import PciamGrid, FLAG_NO_GRAPH
g = synthgrid.make_grid(2, 2, 1040, 1392)
p = PciamGrid(2, 2, 1040, 1392, chunk_pairs=2, chunk_tiles=2, flags=FLAG_NO_GRAPH); p.load_grid(g.tiles); w, n = p.compute_translations()
b = PciamGrid(2, 2, 1040, 1392, chunk_pairs=1, chunk_tiles=1, pool_tiles=4, flags=FLAG_NO_GRAPH)
h = torch.empty(g.tiles.shape, dtype=torch.uint16, pin_memory=True); h.numpy()[...] = g.tiles
b.compute_from_host_async(h, 0); wb, nb = b.get_translations()
assert wb.tobytes() == w.tobytes() and nb.tobytes() == n.tobytes()
s = p.surface(1, 0)
q = PciamGrid(2, 2, 1040, 1392, precision=1); q.load_grid(g.tiles); w2, n2 = q.compute_translations()
assert (w["dx"] == w2["dx"]).all() and (n["dy"] == n2["dy"]).all()
print("big ok (fp32 + bounded pool + surface hook + fp64)", w["dx"].tolist(), n["dy"].tolist())'
for tool in memcheck racecheck synccheck initcheck; do
  echo "== $tool (config 1)"
  timeout 900 compute-sanitizer --tool $tool --print-limit 20 python -c "$SMOKE" 2>&1 | tail -6
done
for tool in memcheck racecheck; do
  echo "== $tool (2x2 @ 1392x1040)"
  timeout 1200 compute-sanitizer --tool $tool --print-limit 20 python -c "$BIG" 2>&1 | tail -6
done
COMPOSE='import numpy as np, torch, synthgrid; from paper_conf_icpp_blattnerkcsbz14_b200 import compose_overlay
for (n, m, H, W, ov) in ((3, 4, 192, 256, 0.1), (3, 4, 26, 58, 0.3)):
    g = synthgrid.make_grid(n, m, H, W, overlap=ov, delta=4, seed=52)
    dev = torch.from_numpy(g.tiles.view(np.int16)).view(torch.uint16).cuda()
    c = compose_overlay(dev, g.origins); torch.cuda.synchronize()
print("compose ok (16-byte and pixel paths)")'
for tool in memcheck initcheck; do
  echo "== $tool (phase 3 overlay)"
  timeout 600 compute-sanitizer --tool $tool --print-limit 20 python -c "$COMPOSE" 2>&1 | tail -4
done
