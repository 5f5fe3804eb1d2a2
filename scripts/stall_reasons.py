"""Top SASS instructions of an ncu source page (csv) with their stall-reason split.
usage: ncu -i rep --page source --csv --print-source sass -k regex:K > x.csv; python scripts/stall_reasons.py x.csv [top]"""
import csv, sys
rows = list(csv.reader(open(sys.argv[1])))
top = int(sys.argv[2]) if len(sys.argv) > 2 else 20
hi = next(i for i, r in enumerate(rows) if r and r[0] == "Address")
h = rows[hi]
si = h.index("Warp Stall Sampling (All Samples)")
st = [i for i, k in enumerate(h) if k.startswith("stall_")]
data = []
for r in rows[hi + 1:]:
    if len(r) <= si or not r[0].startswith("0x"):
        continue
    data.append(r)
tot = sum(float(r[si] or 0) for r in data)
agg = {}
for r in data:
    for i in st:
        agg[h[i]] = agg.get(h[i], 0) + float(r[i] or 0)
print("total samples", tot)
print("by reason:", ", ".join(f"{k[6:]} {100*v/tot:.1f}%" for k, v in sorted(agg.items(), key=lambda kv: -kv[1])[:10]))
for r in sorted(data, key=lambda r: -float(r[si] or 0))[:top]:
    rs = sorted(((h[i][6:], float(r[i] or 0)) for i in st), key=lambda kv: -kv[1])[:3]
    print(f"{100*float(r[si])/tot:5.1f}% {r[0]} {r[1][:60]:60s} " + " ".join(f"{k}:{v:.0f}" for k, v in rs))
