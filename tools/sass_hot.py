"""Top SASS instructions by executed count and by stall samples from an ncu
source page (--page source --csv --print-source=sass)."""
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
h = rows[1]
data = rows[2:]
ie = h.index("Instructions Executed")
ss = h.index("Warp Stall Sampling (All Samples)")
src = h.index("Source")
addr = h.index("Address")
stall_cols = [i for i, x in enumerate(h) if x.startswith("stall_") and "Not Issued" not in x]
def num(x):
    try:
        return float(x)
    except Exception:
        return 0.0
tot_i = sum(num(r[ie]) for r in data)
tot_s = sum(num(r[ss]) for r in data)
print(f"total inst {tot_i:.3e}  total stall samples {tot_s:.0f}")
agg = {}
for r in data:
    for c in stall_cols:
        agg[h[c]] = agg.get(h[c], 0) + num(r[c])
print("stall reasons:", sorted(((round(v / max(tot_s, 1) * 100, 1), k) for k, v in agg.items() if v), reverse=True)[:10])
n = int(sys.argv[2]) if len(sys.argv) > 2 else 25
print("--- top by stall samples")
for r in sorted(data, key=lambda r: -num(r[ss]))[:n]:
    top = sorted(((num(r[c]), h[c]) for c in stall_cols), reverse=True)[:2]
    print(f"{r[addr]:>6s} {num(r[ss]):8.0f} {num(r[ie]):10.0f}  {r[src][:60]:60s} {top}")
