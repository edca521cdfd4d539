import json
import sys
tag = sys.argv[1] if len(sys.argv) > 1 else ""
line = sys.stdin.read().strip()
try:
    d = json.loads(line)
except json.JSONDecodeError:
    print(tag, "FAILED:", line[-500:])
    sys.exit(0)
k = {n: round(v, 2) for n, v in d["roofline"]["kernels_ms_per_step"].items()}
print(tag, f"ms/step={d['ms_per_step']:.2f}", f"pairs/s={d['value']:.0f}",
      f"frac={d['roofline']['frac']:.3f}", k, "clk", d["clocks"].get("sm_mhz"))
