"""Warp-level instructions executed per code phase of an ncu source-page CSV
(--page source --csv --print-source sass): the SASS between barriers, mbarrier waits, warp
syncs and backward branches, with each phase's share of the kernel's instructions and its
top opcodes.  Usage: python tools/inst_phases.py src.csv"""
import collections
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
hi = next(i for i, r in enumerate(rows) if r and r[0] == "Address")
h = rows[hi]
d = rows[hi + 1:]
col = next(c for c in ("Instructions Executed", "Warp Instructions Executed") if c in h)
iE = h.index(col)
tot = sum(float(r[iE] or 0) for r in d)
print(f"total warp instructions {tot:.4g}, SASS lines {len(d)}")
start, s, ops = 0, 0.0, collections.Counter()


def flush(a, b):
    if s > 0:
        top = ", ".join(f"{k}={v / s * 100:.0f}%" for k, v in ops.most_common(5))
        print(f"[{a:5d}-{b:5d}] {s / tot * 100:5.1f}%  {s:.4g}  {top}")


for i, r in enumerate(d):
    n = float(r[iE] or 0)
    src = r[1].strip()
    op = src.split()[0] if src else ""
    if op.startswith("@"):
        op = src.split()[1] if len(src.split()) > 1 else op
    s += n
    ops[op.split(".")[0]] += n
    mark = any(k in src for k in ("BAR", "SYNCS", "WARPSYNC", "REDUX")) or (
        " BRA " in f" {src} " and "0x" in src and i == len(d) - 1)
    if mark or i == len(d) - 1:
        flush(start, i)
        if mark:
            print("       ", src[:70])
        start, s, ops = i + 1, 0.0, collections.Counter()
