"""The SASS instructions with the most warp-stall samples in an ncu source-page CSV.
Usage: python tools/stall_hot.py src.csv [top_n]"""
import csv, sys
rows = list(csv.reader(open(sys.argv[1])))
# find header
hi = next(i for i,r in enumerate(rows) if r and r[0]=="Address")
h = rows[hi]; data = rows[hi+1:]
iS = h.index("Warp Stall Sampling (All Samples)"); iN = h.index("Warp Stall Sampling (Not-issued Samples)")
tot = sum(int(r[iS] or 0) for r in data)
print("total samples", tot, "instrs", len(data))
# group into windows of 'kind'
top = sorted(data, key=lambda r: -int(r[iS] or 0))[:int(sys.argv[2]) if len(sys.argv)>2 else 25]
for r in top:
    print(f"{int(r[iS])/tot*100:5.1f}% {r[iN]:>6} {r[0][-5:]} {r[1].strip()[:90]}")
