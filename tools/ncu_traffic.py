#!/usr/bin/env python3
"""dram__bytes_read.sum + dram__bytes_write.sum per launch of each kernel from the ncu
--set full captures (cold: caches flushed before the launch; warm: --cache-control none).
    python tools/ncu_traffic.py TAG kernel_tag...   (reads gpurun_out/TAG_<k>[_warm].ncu-rep)"""
import csv
import io
import json
import subprocess
import sys

NAMES = {"k1p_fwd": "k1_fwd_rows", "k1w_fwd": "k1_fwd_rows", "k2t_fwd": "k2_fwd_cols",
         "k3t_pair": "k3_pair_cols", "k4w_pair": "k4_pair_rows",
         "k4p_pair": "k4_pair_rows", "k5_ccf": "k5_ccf_moments"}
MUL = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "nsecond": 1e-9, "usecond": 1e-6,
       "msecond": 1e-3, "ns": 1e-9, "us": 1e-6, "ms": 1e-3}


def metrics(rep):
    t = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True,
                       text=True).stdout
    r = list(csv.reader(io.StringIO(t)))
    h, u, v = r[0], r[1], r[2]

    def get(m):
        i = h.index(m)
        return float(v[i]) * MUL.get(u[i], 1)
    return {"dram_read_bytes": get("dram__bytes_read.sum"),
            "dram_write_bytes": get("dram__bytes_write.sum"),
            "duration_s": get("gpu__time_duration.sum")}


def main():
    tag, ks = sys.argv[1], sys.argv[2:]
    out = {}
    for k in ks:
        name = NAMES.get(k, k)
        d = {}
        for variant, suffix in (("cold", ""), ("warm", "_warm")):
            try:
                d[variant] = metrics(f"gpurun_out/{tag}_{k}{suffix}.ncu-rep")
            except Exception as e:  # noqa: BLE001
                d[variant] = {"error": str(e)}
        if "dram_read_bytes" in d["cold"]:
            d["bytes_per_launch"] = d["cold"]["dram_read_bytes"] + d["cold"]["dram_write_bytes"]
        d["note"] = ("dram__bytes_read.sum + dram__bytes_write.sum of one launch, ncu --set full "
                     "(cold: caches flushed before the launch; warm: --cache-control none)")
        out[name] = d
    json.dump(out, sys.stdout, indent=1)


if __name__ == "__main__":
    main()
