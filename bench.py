#!/usr/bin/env python3
"""Benchmark: PCIAM tile-pair translations/sec on the paper's headline 42x59 grid.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config 3] [--impl ours|reference]

A "step" is one pass of the whole hot path (forward
R2C FFT of every tile, NCPS + inverse FFT + argmax + 4-candidate CCF + selection
for every west/north pair) over the synthetic grid of BASELINE.json configs[2]
(42x59 tiles of 1392x1040 uint16).  `value` is pairs/s
with the tiles resident in HBM; `e2e` is the same through the C ABI from pinned
host buffers (H2D of the tiles + D2H of the results inside the timed region).
Inputs (7.2 GB of tiles, 7.3 GB of resident phase spectra) are far larger than the 126 MB L2.

N > 1 (torchrun): row-band partition of the grid, one rank per GPU; each rank
owns tiles [k*nt/N, (k+1)*nt/N) and keeps the preceding tile row resident (halo):
the halo's spectra are received from the previous rank (NCCL send/recv over NVLink,
paper future work P:L1512-1517), its raw pixels are loaded with the band; the per-step
time is the max over ranks (all_reduce MAX).

--impl reference: the reference arm is the oracle (oracle/, plain C, fp64),
timed as it stands on the host cores on a bounded sample of the same workload.
"""
from __future__ import annotations

import argparse
import json
import math
import os
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import synthgrid  # noqa: E402
from paper_conf_icpp_blattnerkcsbz14_b200.parallel import band as parallel_band  # noqa: E402

HBM_SPEC_GBPS = 8000.0             # B200 HBM3e spec (report fractions of both)
PAPER_PAIRS_PER_S = 4855 / 49.7   # Pipelined-GPU, 1x Tesla C2070, Table II: context
REASON_BITS = {0x1: "gpu_idle", 0x2: "applications_clocks_setting", 0x4: "sw_power_cap",
               0x8: "hw_slowdown", 0x10: "sync_boost", 0x20: "sw_thermal_slowdown",
               0x40: "hw_thermal_slowdown", 0x80: "hw_power_brake_slowdown",
               0x100: "display_clock_setting"}


def peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            return json.load(f), "measured"
    except OSError:
        return {"hbm_gbs": 6650.0, "sm_max_mhz": 1965.0}, "fallback"


class ClockSampler:
    """nvidia-smi clocks + throttle reasons sampled every 200 ms during the timed region."""

    def __init__(self, device: int):
        self.device = device
        self.proc = None
        self.lines = []

    def __enter__(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.device),
                 "--query-gpu=clocks.sm,clocks.max.sm,clocks_event_reasons.active",
                 "--format=csv,noheader,nounits", "-lms", "200"],
                stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except OSError:
            self.proc = None
        return self

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    def __exit__(self, *a):
        if self.proc:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except subprocess.TimeoutExpired:
                self.proc.kill()

    def summary(self):
        sm, mx, reasons = [], None, set()
        for ln in self.lines:
            parts = [p.strip() for p in ln.split(",")]
            if len(parts) < 3:
                continue
            try:
                sm.append(float(parts[0]))
                mx = float(parts[1])
                bits = int(parts[2], 16)
            except ValueError:
                continue
            for b, name in REASON_BITS.items():
                if bits & b and name != "gpu_idle":
                    reasons.add(name)
        if not sm:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": [], "samples": 0}
        return {"sm_mhz": float(np.median(sm)), "sm_max_mhz": mx, "reasons": sorted(reasons),
                "samples": len(sm)}


def band(rank: int, world: int, n: int, m: int):
    nt = n * m
    b, e = rank * nt // world, (rank + 1) * nt // world
    halo = max(0, b - m)
    return b, e, halo


# The oracle's bounded sample (cpu_baseline and the reference arm time the same one): the
# top-left 4 x c corner of the workload's grid -- the same tiles and pair kinds as the GPU
# step -- through oracle.grid (fp64, Fig. 4 over Fig. 2) on every host core; c is chosen so the
# corner holds about two tiles per core (the oracle's forward phase spreads tiles over threads),
# i.e. a few seconds of work per sample.


def sub_grid():
    cores = os.cpu_count() or 1
    return 4, max(3, round(2 * cores / 4))


def metric_name(cfg: dict) -> str:
    """One metric string for both arms (the driver pairs them by it)."""
    return f"tile-pair translations/sec ({cfg['name']} grid)"


def workload_config(cfg: dict, config_index: int) -> dict:
    n, m, H, W = cfg["n"], cfg["m"], cfg["H"], cfg["W"]
    return {"workload": f"{cfg['name']} (BASELINE.json configs[{config_index - 1}])",
            "grid": f"{n}x{m}", "tile": f"{W}x{H} uint16", "pairs": 2 * n * m - n - m,
            "tiles": n * m, "overlap": cfg["overlap"], "seed": synthgrid.SEED}


def oracle_sample(cfg: dict):
    r, c = sub_grid()
    g = synthgrid.make_grid(r, c, cfg["H"], cfg["W"], overlap=cfg["overlap"],
                            delta=cfg["delta"])
    pairs = 2 * r * c - r - c
    desc = (f"{r}x{c} corner of the {cfg['name']} grid ({pairs} pairs, "
            f"{r * c} forward transforms) per sample, oracle.grid fp64")
    return g, pairs, desc


def cpu_baseline(cfg: dict):
    """The oracle as it stands, on the bounded sample, all host cores (one sample)."""
    import oracle
    g, pairs, desc = oracle_sample(cfg)
    cores = os.cpu_count() or 1
    t = time.perf_counter()
    oracle.grid(g.tiles, threads=cores)
    dt = time.perf_counter() - t
    return {"value": pairs / dt, "unit": "pairs/s", "cores": cores, "kind": "oracle",
            "sample": f"{desc}, {dt:.1f} s wall"}


def run_reference(args, cfg):
    """Reference arm: the oracle timed on the host cores, the same bounded sample per step."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    import oracle
    g, pairs, desc = oracle_sample(cfg)
    cores = os.cpu_count() or 1
    for _ in range(args.warmup):
        oracle.grid(g.tiles, threads=cores)
    t = time.perf_counter()
    for _ in range(args.steps):
        oracle.grid(g.tiles, threads=cores)
    dt = time.perf_counter() - t
    value = pairs * args.steps / dt
    conf = workload_config(cfg, args.config)
    conf["sample"] = desc
    line = {
        "impl": "reference", "metric": metric_name(cfg),
        "value": value, "unit": "pairs/s", "n_gpus": args.gpus, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": 1e3 * dt / args.steps, "higher_is_better": True,
        "scaling": "strong", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
        "config": conf,
        "cpu_baseline": {"value": value, "unit": "pairs/s", "cores": cores, "kind": "oracle",
                         "sample": desc},
        "e2e": {"value": value, "unit": "pairs/s", "h2d_bytes_per_step": 0,
                "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)


def run_stream(args, cfg):
    """configs[3]: the time series (161 scans x 2 channels of 18x22 grids) streamed through
    bounded grid slots (stream.py): every grid's H2D from pinned host
    memory, steps 2-7 and the D2H of its results are inside the timed region (host clock),
    whole grids dealt round-robin to the ranks.  A bounded sample of the series is timed
    (--ts-grids); its tiles cycle through P distinct pre-generated scans/channels."""
    import torch
    import torch.distributed as dist

    from paper_conf_icpp_blattnerkcsbz14_b200.stream import GridStream, shard
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    torch.cuda.set_device(local)
    if world > 1:
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    n, m, H, W = cfg["n"], cfg["m"], cfg["H"], cfg["W"]
    series = [(s, c) for s in range(cfg["scans"]) for c in range(cfg["channels"])]
    P = 4
    pool = []
    for i in range(P):
        s, c = series[i]
        t = torch.empty((n, m, H, W), dtype=torch.uint16, pin_memory=True)
        synthgrid.make_grid(n, m, H, W, overlap=cfg["overlap"], delta=cfg["delta"], scan=s,
                            channel=c, out=t.numpy())
        pool.append(t)
    total = min(args.ts_grids, len(series))
    mine_w = shard(list(range(args.warmup)), rank, world)
    mine = shard(list(range(total)), rank, world)
    with GridStream(n, m, H, W, slots=args.ts_slots, device=local,
                    chunk_pairs=args.chunk_pairs, chunk_tiles=args.chunk_tiles) as gs:
        fill = (lambda i, host: pool[i % P])
        gs.run(mine_w, fill)
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()
        with ClockSampler(local) as clk:
            t0 = time.perf_counter()
            done = gs.run(mine, fill)
            torch.cuda.synchronize()
            dt = time.perf_counter() - t0
        ppg = gs.pairs_per_grid
    if world > 1:
        tt = torch.tensor([dt, float(done)], dtype=torch.float64, device="cuda")
        mx = tt.clone()
        dist.all_reduce(mx, op=dist.ReduceOp.MAX)
        dist.all_reduce(tt, op=dist.ReduceOp.SUM)
        dt, done = float(mx[0].item()), int(tt[1].item())
    pairs = done * ppg
    if rank == 0:
        line = {
            "metric": f"tile-pair translations/sec ({cfg['name']} time series, streamed)",
            "value": pairs / dt, "unit": "pairs/s", "n_gpus": world, "steps": total,
            "warmup": args.warmup, "ms_per_step": 1e3 * dt / max(1, total // world),
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f32",
            "data": "synthetic",
            "config": {"workload": f"{cfg['name']} (BASELINE.json configs[3]), sample of "
                                   f"{total} of {len(series)} grids",
                       "grid": f"{n}x{m}", "tile": f"{W}x{H} uint16", "slots": args.ts_slots,
                       "pairs_per_grid": ppg, "parallelism": f"whole grids round-robin x{world}",
                       "step": "one grid: H2D + steps 2-7 + D2H"},
            "e2e": {"value": pairs / dt, "unit": "pairs/s",
                    "h2d_bytes_per_step": n * m * H * W * 2, "d2h_bytes_per_step": ppg * 64,
                    "h2d_GBps": done * n * m * H * W * 2 / dt / 1e9 / max(1, world)},
            "clocks": clk.summary(),
        }
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()


def run_pooled(args, cfg):
    """Bounded mode (stitch_config.pool_tiles): the grid streams from pinned host
    memory through a fixed pool of tile slots recycled by reference count, so device memory
    no longer grows with the grid.  Every step includes the H2D of all tiles (the pool cannot
    keep them), so `value` is device-timed steps 1-7 (CUDA events on the library stream) and
    e2e adds the results' D2H on the host clock."""
    import torch

    from paper_conf_icpp_blattnerkcsbz14_b200 import PciamGrid
    n, m, H, W = cfg["n"], cfg["m"], cfg["H"], cfg["W"]
    torch.cuda.set_device(0)
    host = torch.empty((n, m, H, W), dtype=torch.uint16, pin_memory=True)
    synthgrid.make_grid(n, m, H, W, overlap=cfg["overlap"], delta=cfg["delta"],
                        out=host.numpy().view(np.uint16))
    pg = PciamGrid(n, m, H, W, pool_tiles=args.pool, chunk_pairs=args.chunk_pairs,
                   chunk_tiles=args.chunk_tiles)
    ws = pg._ws.numel()
    for _ in range(max(1, args.warmup)):
        pg.compute_from_host_async(host, 0)
    pg.synchronize()
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with ClockSampler(0) as clk:
        ev0.record(pg.stream)
        for _ in range(args.steps):
            pg.compute_from_host_async(host, 0)
        ev1.record(pg.stream)
        torch.cuda.synchronize()
    ms = ev0.elapsed_time(ev1) / args.steps
    t0 = time.perf_counter()
    for _ in range(max(1, args.e2e_steps)):
        pg.compute_from_host_async(host, 0)
        west, north = pg.get_translations()
    e2e_s = (time.perf_counter() - t0) / max(1, args.e2e_steps)
    o = synthgrid.origins(n, m, H, W, cfg["overlap"], cfg["delta"])
    exact = bool(np.array_equal(west["dx"][:, 1:], o[:, 1:, 0] - o[:, :-1, 0]) and
                 np.array_equal(north["dy"][1:], o[1:, :, 1] - o[:-1, :, 1]))
    pairs = 2 * n * m - n - m
    import paper_conf_icpp_blattnerkcsbz14_b200 as pkg
    resident = pkg.workspace_size(pkg.make_config(n, m, H, W))
    conf = workload_config(cfg, args.config)
    conf.update({"mode": f"bounded pool of {args.pool} tile slots (stitch_config.pool_tiles)",
                 "workspace_GB": ws / 1e9, "resident_workspace_GB": resident / 1e9,
                 "grid_wall_ms": ms, "shifts_recovered": exact})
    line = {"metric": metric_name(cfg), "value": pairs / (ms / 1e3), "unit": "pairs/s",
            "n_gpus": 1, "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms,
            "higher_is_better": True, "scaling": "strong", "vs_baseline": None,
            "dtype": "f32 (Q15 resident phasor, fp16 Q intermediate)" if W >= 1024
                     else "f32 (Q15 resident phasor)", "data": "synthetic", "config": conf,
            "e2e": {"value": pairs / e2e_s, "unit": "pairs/s",
                    "h2d_bytes_per_step": n * m * H * W * 2, "d2h_bytes_per_step": pairs * 64,
                    "grid_wall_ms": e2e_s * 1e3},
            "gpu_launches": pg.last_counts()["launches"] * args.steps,
            "clocks": clk.summary()}
    pg.close()
    print(json.dumps(line), flush=True)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=30)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--config", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--chunk-pairs", type=int, default=0)
    ap.add_argument("--chunk-tiles", type=int, default=0)
    ap.add_argument("--e2e-steps", type=int, default=3)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--compose", action="store_true",
                    help="also time phase 2 (positions) and phase 3 (overlay composite)")
    ap.add_argument("--ts-grids", type=int, default=24, help="config 4: grids streamed (timed)")
    ap.add_argument("--ts-slots", type=int, default=2, help="config 4: grid slots in flight")
    ap.add_argument("--precision", default="f32", choices=["f32", "f64"],
                    help="arithmetic of steps 2-5 (f64: the optional fp64 path, SURVEY 8 f2)")
    ap.add_argument("--dist-backend", default="nccl", choices=["nccl", "gloo"],
                    help="gloo: logic check of the N > 1 path with ranks sharing GPUs (not a "
                         "bench number; the halo goes through host memory)")
    ap.add_argument("--pool", type=int, default=0,
                    help="bounded mode: stream the grid from pinned host memory through this "
                         "many tile slots (SURVEY 8 f1)")
    ap.add_argument("--transport", default=None, choices=["library", "torch", "recompute"],
                    help="N > 1 halo: the library's NCCL send/recv (default with nccl), "
                         "torch.distributed on a side stream (default with gloo), or recompute")
    args = ap.parse_args()
    cfg = dict(synthgrid.CONFIGS[args.config])
    if args.impl == "reference":
        return run_reference(args, cfg)
    if args.config == 4:
        return run_stream(args, cfg)
    if args.pool > 0:
        return run_pooled(args, cfg)

    import torch
    import torch.distributed as dist

    from paper_conf_icpp_blattnerkcsbz14_b200 import StitchError
    from paper_conf_icpp_blattnerkcsbz14_b200.parallel import BandPciam, gather_translations

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if world != args.gpus:
        raise SystemExit(f"--gpus {args.gpus} but WORLD_SIZE={world}")
    if args.dist_backend == "gloo":
        # logic check of the multi-rank path on fewer GPUs than ranks: ranks share devices,
        # the halo exchange stages through host memory (parallel.exchange_halo)
        local = local % torch.cuda.device_count()
    torch.cuda.set_device(local)
    if world > 1:
        if args.dist_backend == "nccl":
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
        else:
            dist.init_process_group("gloo")
    red_dev = "cuda" if args.dist_backend == "nccl" else "cpu"

    n, m, H, W = cfg["n"], cfg["m"], cfg["H"], cfg["W"]
    b, e, halo = band(rank, world, n, m)
    r0, r1 = halo // m, (e - 1) // m + 1            # tile rows this rank holds
    assert (r0, r1) == (parallel_band(rank, world, n, m).row_begin,
                        parallel_band(rank, world, n, m).row_end)
    # host tiles of the rows this rank needs, in pinned memory (the e2e source buffer)
    host = torch.empty((r1 - r0, m, H, W), dtype=torch.uint16, pin_memory=True)
    synthgrid.make_grid(n, m, H, W, overlap=cfg["overlap"], delta=cfg["delta"],
                        out=host.numpy().view(np.uint16), rows=(r0, r1))
    first = r0 * m

    transport = args.transport or ("library" if args.dist_backend == "nccl" else "torch")
    kw = dict(chunk_pairs=args.chunk_pairs, chunk_tiles=args.chunk_tiles,
              precision=1 if args.precision == "f64" else 0)
    try:
        bp = BandPciam(n, m, H, W, rank, world, device=local, transport=transport, **kw)
    except StitchError as err:
        # the library's NCCL communicator could not be formed (stitch_init is collective, so
        # every rank lands here): measure with the torch.distributed transport instead, and say so
        if transport != "library":
            raise
        print(f"bench: library NCCL transport unavailable ({err}); using torch.distributed",
              file=sys.stderr, flush=True)
        transport = "torch"
        bp = BandPciam(n, m, H, W, rank, world, device=local, transport=transport, **kw)
    pg = bp.grid
    stream = pg.stream          # the stream the library enqueues on (events must be recorded here)
    pg.load_tiles(host, first)
    pg.synchronize()
    pairs_local = pg.npairs

    def barrier():
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()

    def max_over_ranks(x: float) -> float:
        if world == 1:
            return x
        t = torch.tensor([x], dtype=torch.float64, device=red_dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        return float(t.item())

    def sum_over_ranks(x: float) -> float:
        if world == 1:
            return x
        t = torch.tensor([x], dtype=torch.float64, device=red_dev)
        dist.all_reduce(t, op=dist.ReduceOp.SUM)
        return float(t.item())

    # ---- warm-up, then K timed steps with tiles resident in HBM ----------------------------
    for _ in range(args.warmup):
        bp.step_async()
    barrier()
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    launches = 0
    with ClockSampler(local) as clk:
        barrier()
        ev0.record(stream)
        for _ in range(args.steps):
            bp.step_async()
            launches += pg.last_counts()["launches"]
        ev1.record(stream)
        barrier()
    dev_ms = ev0.elapsed_time(ev1) / args.steps
    ms = max_over_ranks(dev_ms)
    total_pairs = sum_over_ranks(pairs_local)
    value = total_pairs / (ms / 1e3)
    clocks = clk.summary()

    # ---- per-kernel durations (timing mode 2: an event after every launch) ---------------
    pg.set_timing(2)
    kt_sum = {}
    for _ in range(max(1, min(args.steps, 5))):
        bp.step_async()
        pg.synchronize()
        for k, v in pg.kernel_timings().items():
            s = kt_sum.setdefault(k, {"ms": 0.0, "launches": 0})
            s["ms"] += v["ms"]
            s["launches"] += v["launches"]
    pg.set_timing(0)
    step_kernel_ms = sum(v["ms"] for v in kt_sum.values())
    dom = max(kt_sum, key=lambda k: kt_sum[k]["ms"])
    S = H * (W // 2 + 1) * 8          # fp32 complex half spectrum (kx in [0, W/2]) bytes
    T = H * W * 2                     # raw tile bytes
    # Algorithmic bytes per unit (tile or pair) of each kernel in this design (DESIGN.md
    # "Roofline"): what it must read + write at least once; the resident spectrum is a
    # 4-byte phase code per bin (S/2), intermediates G and Q are complex (S).
    alg_bytes_per_unit = {
        "k1_fwd_rows": T + S,          # raw in, row-transformed G out
        "k2_fwd_cols": S + S // 2,     # G in, phase spectrum out
        "k3_pair_cols": S // 2 * 2 + S,  # two phase spectra in, Q out
        "k4_pair_rows": S,             # Q in (the surface is never stored)
        "k5_ccf_moments": 2 * T,       # the four candidate overlaps of A and B (HW pixels each)
        "k6_finalize": 8 + 160 + 64}
    q_half = W >= 1024 and args.precision != "f64"   # Plan::Q_HALF: Q as scaled fp16 pairs
    if q_half:
        alg_bytes_per_unit.update({"k3_pair_cols": S // 2 * 2 + S // 2, "k4_pair_rows": S // 2})
    if args.precision == "f64":
        # fp64 path (D1..D4, pciam_fp64.cuh): complex intermediates are 2S (complex128), the
        # resident unit phasor is S (Q31, 8 B per bin); D4's per-block argmax partials are ~0
        alg_bytes_per_unit.update({"k1_fwd_rows": T + 2 * S, "k2_fwd_cols": 3 * S,
                                   "k3_pair_cols": 4 * S, "k4_pair_rows": 2 * S})
    kd = kt_sum[dom]
    nsteps_k = max(1, min(args.steps, 5))
    fwd_tiles = (e - b) if bp.use_exchange else (e - halo)   # halo received or recomputed
    units_total = {"k1_fwd_rows": fwd_tiles, "k2_fwd_cols": fwd_tiles,
                   "k3_pair_cols": pairs_local, "k4_pair_rows": pairs_local,
                   "k5_ccf_moments": pairs_local, "k6_finalize": pairs_local}
    bytes_per_launch = alg_bytes_per_unit[dom] * units_total[dom] / (kd["launches"] / nsteps_k)
    avg_launch_ms = kd["ms"] / kd["launches"]
    pk, pk_kind = peaks()
    achieved = bytes_per_launch / (avg_launch_ms / 1e3) / 1e9
    kms = {k: v["ms"] / nsteps_k for k, v in kt_sum.items()}
    klaunch = {k: v["launches"] / nsteps_k for k, v in kt_sum.items()}
    roofline = {"bound": "hbm", "kernel": dom, "achieved": achieved, "peak": pk["hbm_gbs"],
                "unit": "GB/s", "frac": achieved / pk["hbm_gbs"], "traffic": None,
                "peak_source": pk_kind, "avg_launch_ms": avg_launch_ms,
                "alg_bytes_per_launch": bytes_per_launch,
                "byte_model": ("design: bytes each kernel must move with the resident spectrum "
                               "as a Q15 unit phasor (S/2 per tile), complex64 G chunks (S) and "
                               + ("fp16 Q chunks (S/2)" if q_half else "complex64 Q chunks (S)")
                               + "; DESIGN.md section 6"),
                "share_of_step": kd["ms"] / step_kernel_ms,
                "kernels_ms_per_step": kms,
                "kernels_launches_per_step": klaunch,
                # algorithmic GB/s per kernel (K5's 2T per pair re-reads tiles K1 left in L2,
                # so it is not an HBM fraction: see kernels_dram_frac)
                "kernels_alg_GBps": {k: alg_bytes_per_unit[k] * units_total[k] / (ms / 1e3) / 1e9
                                     for k, ms in kms.items() if ms > 0}}
    design_bytes = sum(alg_bytes_per_unit[k] * units_total[k] for k in alg_bytes_per_unit)
    survey_2pass = fwd_tiles * (T + 3 * S) + pairs_local * (4 * S + 2 * T)
    roofline["step_alg_GBps"] = design_bytes / (dev_ms / 1e3) / 1e9
    roofline["step_frac"] = roofline["step_alg_GBps"] / pk["hbm_gbs"]
    roofline["survey_2pass_GBps"] = survey_2pass / (dev_ms / 1e3) / 1e9
    roofline["spec_frac"] = roofline["step_alg_GBps"] / HBM_SPEC_GBPS       # vs the ~8 TB/s spec
    # FFT FLOP/s (north_star "FFT FLOP/s against the fp32 peak"): the nominal
    # 2.5 N log2 N per real 2-D transform (N = HW), one per tile (forward) and one per pair
    # (inverse), against 2 FLOP x 128 FP32 lanes x SMs x the SM clock measured under load
    # whole job: every rank's transforms (halo rows recomputed without the exchange count too)
    nominal = 2.5 * H * W * math.log2(H * W) * sum_over_ranks(fwd_tiles + pairs_local)
    sm_mhz = clocks.get("sm_mhz") or pk.get("sm_max_mhz", 1965.0)
    n_sm = torch.cuda.get_device_properties(local).multi_processor_count
    fp_peak = 2 * 128 * n_sm * sm_mhz * 1e6 / 1e12
    fft = {"nominal_flop_per_step": nominal, "achieved_tflops": nominal / (dev_ms / 1e3) / 1e12,
           "peak_tflops": fp_peak, "peak": "fp64" if args.precision == "f64" else "fp32",
           "sm_mhz": sm_mhz, "convention": "2.5 N log2 N per real 2-D transform, N = H*W"}
    if args.precision == "f64":   # B200 FP64 vector rate: half the FP32 rate
        fft["peak_tflops"] = fp_peak / 2
    fft["frac"] = fft["achieved_tflops"] / fft["peak_tflops"]
    # Measured DRAM traffic: dram__bytes_read.sum + dram__bytes_write.sum of one launch of each
    # kernel (ncu --set full, caches flushed before the launch: an upper bound for a step
    # whose kernels share L2) at the default chunks, scaled by the launches per step; the
    # HBM fraction of each kernel and of the step on those bytes.
    traffic_path = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    default_chunks = args.chunk_pairs == 0 and args.chunk_tiles == 0
    if os.path.exists(traffic_path) and args.precision == "f32" and default_chunks:
        with open(traffic_path) as f:
            tj = json.load(f)
        tr = tj.get(dom)
        if tr:
            roofline["traffic"] = tr.get("bytes_per_launch")
        dram = {k: tj[k]["bytes_per_launch"] * klaunch[k] for k in kms
                if k in tj and kms[k] > 0}
        roofline["dram_source"] = tj.get("_source", "profiles/ncu_traffic.json")
        roofline["kernels_dram_GB_per_step"] = {k: v / 1e9 for k, v in dram.items()}
        roofline["kernels_dram_frac"] = {k: v / (kms[k] / 1e3) / 1e9 / pk["hbm_gbs"]
                                         for k, v in dram.items()}
        roofline["dram_frac"] = (dram[dom] / (kms[dom] / 1e3) / 1e9 / pk["hbm_gbs"]
                                 if dom in dram else None)
        roofline["step_dram_GB"] = sum(dram.values()) / 1e9
        roofline["step_dram_frac"] = sum(dram.values()) / (dev_ms / 1e3) / 1e9 / pk["hbm_gbs"]

    # ---- e2e: through the C ABI from pinned host buffers ------------------------------
    e2e_steps = max(1, args.e2e_steps)
    pipelined = bp.transport != "torch"       # one library call per step: H2D pipelined
    if pipelined:
        pg.compute_from_host_async(host, first)     # warm: captures this buffer's graph
        pg.get_translations()
    barrier()
    t0 = time.perf_counter()
    for _ in range(e2e_steps):
        if pipelined:   # per chunk: H2D of its tiles, then its transforms (stitch.h)
            pg.compute_from_host_async(host, first)
        else:
            pg.load_tiles(host, first)              # H2D of this rank's tile rows
            bp.step_async()
        west, north = pg.get_translations()         # D2H of the results, synchronous
    torch.cuda.synchronize()
    e2e_s = max_over_ranks((time.perf_counter() - t0) / e2e_steps)
    h2d = sum_over_ranks((e - halo) * T)          # whole job: every rank's tile rows
    d2h = sum_over_ranks(pairs_local * 64)

    # ---- every rank's translations merged and checked against the generator's known shifts --
    if world > 1:
        west, north = gather_translations(west, north, bp.bd)
    truth_o = synthgrid.origins(n, m, H, W, cfg["overlap"], cfg["delta"])
    shifts_ok = bool(np.array_equal(west["dx"][:, 1:], truth_o[:, 1:, 0] - truth_o[:, :-1, 0]) and
                     np.array_equal(west["dy"][:, 1:], truth_o[:, 1:, 1] - truth_o[:, :-1, 1]) and
                     np.array_equal(north["dx"][1:], truth_o[1:, :, 0] - truth_o[:-1, :, 0]) and
                     np.array_equal(north["dy"][1:], truth_o[1:, :, 1] - truth_o[:-1, :, 1]))

    # ---- optional: stitching phases 2 + 3 on the result (NEXT rows f3, f4) -------------
    phase23 = None
    if args.compose and world == 1:
        from paper_conf_icpp_blattnerkcsbz14_b200 import compose_overlay, global_positions
        t0 = time.perf_counter()
        pos, _ = global_positions(west, north)
        t_p2 = time.perf_counter() - t0
        dev_tiles = torch.empty((n, m, H, W), dtype=torch.uint16, device="cuda")
        dev_tiles.copy_(host)
        canvas = compose_overlay(dev_tiles, pos)            # warm (allocates the canvas)
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        compose_overlay(dev_tiles, pos, canvas)
        torch.cuda.synchronize()
        t_p3 = time.perf_counter() - t0
        # device time of the stream-ordered overlay, REPS back to back (CUDA events)
        reps = 5
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for _ in range(reps):
            compose_overlay(dev_tiles, pos, canvas, sync=False)
        e1.record()
        torch.cuda.synchronize()
        k_p3 = e0.elapsed_time(e1) / reps
        # algorithmic bytes: every covered canvas pixel written once and its tile pixel read once
        covered = int((canvas != 0).sum().item())
        truth = synthgrid.origins(n, m, H, W, cfg["overlap"], cfg["delta"])
        p3_GBps = 2 * 2 * covered / (k_p3 * 1e-3) / 1e9
        phase23 = {"phase2_ms": t_p2 * 1e3, "phase3_ms": t_p3 * 1e3,
                   "phase3_device_ms": k_p3, "phase3_alg_GBps": p3_GBps,
                   "phase3_hbm_frac": p3_GBps / pk["hbm_gbs"],
                   "canvas": list(canvas.shape), "canvas_GB": canvas.numel() * 2 / 1e9,
                   "positions_exact": bool(np.array_equal(pos, truth - truth[0, 0]))}
        del canvas, dev_tiles

    # ---- oracle on the host cores (rank 0, N = 1 only) ----------------------------------
    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        cpu = cpu_baseline(cfg)

    if rank == 0:
        conf = workload_config(cfg, args.config)
        conf.update({"pairs": int(total_pairs), "grid_wall_ms": ms,
                     "parallelism": f"row-bands x{world}",
                     "halo": ({"library": "nccl-exchange (in library)",
                               "torch": "exchange (torch.distributed)"}.get(bp.transport,
                                                                            "recompute")
                              if world > 1 else "none"),
                     "l2": "inputs larger than L2 (7.2 GB tiles, 7.3 GB spectra vs 126 MB)",
                     "shifts_recovered": shifts_ok})
        line = {
            "metric": metric_name(cfg),
            "value": value, "unit": "pairs/s", "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True,
            "scaling": "strong",
            "vs_baseline": value / PAPER_PAIRS_PER_S if args.config == 3 else None,
            "vs_baseline_ref": "BASELINE.md: paper Pipelined-GPU 1x C2070, 42x59 in 49.7 s "
                               "(Table II, P:L1208) = 97.7 pairs/s; other hardware, end to end "
                               "incl. TIFF reads",
            "dtype": ("f64 (Q31 resident phasor)" if args.precision == "f64"
                      else "f32 (Q15 resident phasor, fp16 Q intermediate)" if W >= 1024
                      else "f32 (Q15 resident phasor)"),
            "data": "synthetic",
            "config": conf,
            "roofline": roofline,
            "fft_flops": fft,
            "cpu_baseline": cpu,
            "e2e": {"value": total_pairs / e2e_s, "unit": "pairs/s", "h2d_bytes_per_step": h2d,
                    "d2h_bytes_per_step": d2h, "grid_wall_ms": e2e_s * 1e3,
                    "h2d_GBps": h2d / e2e_s / 1e9,
                    "api": ("stitch_compute_translations_from_host_async (H2D pipelined per "
                            "forward chunk) + stitch_get_translations" if pipelined else
                            "stitch_load_tiles + step + stitch_get_translations")},
            "gpu_launches": launches,
            "clocks": clocks,
        }
        if phase23 is not None:
            line["phase23"] = phase23
        print(json.dumps(line), flush=True)
    bp.close()
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
