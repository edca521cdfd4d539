#!/usr/bin/env python3
"""Summarise ncu reports: key throughput / stall / pipe metrics and the SASS opcode mix.
    python tools/ncu_summary.py gpurun_out/r01b_k3_pair_cols.ncu-rep [...]"""
import collections
import csv
import io
import subprocess
import sys

KEYS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "lts__t_bytes.sum",
        "sm__throughput.avg.pct_of_peak_sustained_elapsed", "launch__registers_per_thread",
        "launch__occupancy_limit_shared_mem", "launch__occupancy_limit_registers",
        "sm__warps_active.avg.pct_of_peak_sustained_active", "smsp__inst_executed.sum",
        "smsp__issue_active.avg.pct_of_peak_sustained_active",
        "sm__inst_executed_pipe_fma.avg.pct_of_peak_sustained_active",
        "sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active",
        "sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active",
        "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum",
        "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum",
        "sm__cycles_elapsed.avg.per_second"]


def raw(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True,
                         text=True).stdout
    r = list(csv.reader(io.StringIO(out)))
    return r[0], r[1], r[2]


def main():
    for rep in sys.argv[1:]:
        h, u, v = raw(rep)
        print(f"== {rep}")
        for k in KEYS:
            if k in h:
                i = h.index(k)
                print(f"  {k:66s} {v[i]:>16s} {u[i]}")
        # counted FP32 FLOP rate (fadd + fmul + 2 ffma per thread instruction) vs the FFMA peak
        fk = {k: f"smsp__sass_thread_inst_executed_op_{k}_pred_on.sum.per_cycle_elapsed"
              for k in ("fadd", "fmul", "ffma")}
        pk = "sm__sass_thread_inst_executed_op_ffma_pred_on.sum.peak_sustained"
        if all(x in h for x in fk.values()) and pk in h:
            fl = sum(float(v[h.index(fk[k])]) * (2 if k == "ffma" else 1) for k in fk)
            peak = 2 * float(v[h.index(pk)])
            print(f"  fp32 FLOP/cycle (fadd+fmul+2ffma) {fl:.0f} of peak {peak:.0f} = {fl / peak:.3f}")
        stalls = [(float(v[i]), h[i]) for i in range(len(h))
                  if h[i].startswith("smsp__average_warps_issue_stalled_")
                  and h[i].endswith("_per_issue_active.ratio") and v[i]]
        stalls.sort(reverse=True)
        print("  stalls/issue:", ", ".join(f"{n.split('stalled_')[1].split('_per')[0]}={x:.2f}"
                                          for x, n in stalls[:7]))
        out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source=sass"],
                             capture_output=True, text=True).stdout
        rows = list(csv.reader(io.StringIO(out)))
        if len(rows) > 2:
            hh = rows[1]
            iS, iE = hh.index("Source"), hh.index("Instructions Executed")
            op = collections.Counter()
            for r in rows[2:]:
                try:
                    n = int(r[iE] or 0)
                except (ValueError, IndexError):
                    continue
                t = r[iS].split()
                if not t:
                    continue
                mn = t[1] if t[0].startswith("@") and len(t) > 1 else t[0]
                op[mn.split(".")[0]] += n
            tot = sum(op.values())
            print("  opcode mix:", ", ".join(f"{k} {100 * c / tot:.1f}%" for k, c in op.most_common(12)))


if __name__ == "__main__":
    main()
