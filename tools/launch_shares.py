#!/usr/bin/env python3
"""Per-kernel share of one step from an ncu launch list (gpu__time_duration.sum per launch).
    python tools/launch_shares.py gpurun_out/r01_launches.csv
ncu times are cold-cache and serialised: compare the SHARES with bench.py's live per-kernel
event timings, not the absolute values."""
import collections
import csv
import re
import sys


def main(path):
    rows = [r for r in csv.reader(open(path)) if len(r) > 10 and r[0].isdigit()]
    tot = collections.Counter()
    cnt = collections.Counter()
    unit = "?"
    for r in rows:
        name = re.sub(r"<.*", "", r[4]).replace("void ", "").strip()
        unit = r[13]
        v = float(r[14].replace(",", ""))
        tot[name] += v
        cnt[name] += 1
    allt = sum(tot.values())
    print(f"launches: {len(rows)}   total device time: {allt:.1f} {unit}")
    print(f"{'kernel':24s} {'launches':>8s} {'total':>12s} {'avg':>10s} {'share':>7s}")
    for k, v in tot.most_common():
        print(f"{k:24s} {cnt[k]:8d} {v:12.1f} {v / cnt[k]:10.2f} {100 * v / allt:6.1f}%")


if __name__ == "__main__":
    main(sys.argv[1])
