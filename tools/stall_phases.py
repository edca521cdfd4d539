"""Warp-stall samples of an ncu source-page CSV (--page source --csv --print-source sass), summed
over the SASS between barriers / mbarrier waits (or every N instructions), with the top stall
reasons of each phase.  Usage: python tools/stall_phases.py src.csv [N]"""
import csv,sys
rows=list(csv.reader(open(sys.argv[1])))
hi=next(i for i,r in enumerate(rows) if r and r[0]=="Address")
h=rows[hi]; d=rows[hi+1:]
iS=h.index('Warp Stall Sampling (All Samples)')
reasons=[x for x in h if x.startswith('stall_') and 'Not Issued' not in x]
ri=[h.index(x) for x in reasons]
tot=sum(int(r[iS] or 0) for r in d)
segstart=0; acc={x:0 for x in reasons}; s=0
def flush(a,b,acc,s):
    top=sorted(acc.items(), key=lambda kv:-kv[1])[:4]
    print(f"[{a:4d}-{b:4d}] {s/tot*100:5.1f}% ", ", ".join(f"{k[6:]}={v/tot*100:.1f}" for k,v in top if v))
for i,r in enumerate(d):
    s+=int(r[iS] or 0)
    for x,j in zip(reasons,ri): acc[x]+=int(r[j] or 0)
    src=r[1]
    if 'BAR' in src or 'SYNCS' in src or i==len(d)-1 or (i-segstart)>=int(sys.argv[2] if len(sys.argv)>2 else 300):
        flush(segstart,i,acc,s)
        if 'BAR' in src or 'SYNCS' in src: print("      ", src.strip()[:60])
        segstart=i+1; s=0; acc={x:0 for x in reasons}
