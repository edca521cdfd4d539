"""bench.py's reference arm runs on the host alone (no GPU): its JSON line has the contract's keys
and the same metric string, unit and direction as the GPU arm, so the driver can pair them."""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_reference_arm_json_line():
    out = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--impl", "reference",
                          "--steps", "1", "--warmup", "0"], capture_output=True, text=True,
                         timeout=600, cwd=ROOT)
    assert out.returncode == 0, out.stderr[-2000:]
    line = json.loads([ln for ln in out.stdout.splitlines() if ln.startswith("{")][-1])
    sys.path.insert(0, ROOT)
    import bench
    import synthgrid
    cfg = dict(synthgrid.CONFIGS[3])
    assert line["impl"] == "reference"
    assert line["metric"] == bench.metric_name(cfg)
    assert line["unit"] == "pairs/s" and line["higher_is_better"] is True
    assert line["value"] > 0 and line["steps"] == 1 and line["warmup"] == 0
    assert line["config"]["workload"] == bench.workload_config(cfg, 3)["workload"]
    assert line["e2e"]["h2d_bytes_per_step"] == 0 and line["e2e"]["d2h_bytes_per_step"] == 0
    cb = line["cpu_baseline"]
    assert cb["kind"] == "oracle" and cb["cores"] >= 1 and cb["value"] == line["value"]
    r, c = bench.sub_grid()
    assert f"{r}x{c} corner" in cb["sample"] and f"{2 * r * c - r - c} pairs" in cb["sample"]
