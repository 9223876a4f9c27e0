"""Top SASS lines by warp-stall samples with their dominant reasons (ncu source page CSV)."""
import csv, sys
rows = list(csv.reader(open(sys.argv[1])))
h = rows[1]; data = rows[2:]
si = h.index("Warp Stall Sampling (All Samples)"); ex = h.index("Instructions Executed")
reasons = [(i, n) for i, n in enumerate(h) if n.startswith("stall_") and "Not Issued" not in n]
tot = sum(int(r[si]) for r in data if r[si].isdigit())
agg = {}
for r in data:
    for i, n in reasons:
        if r[i].isdigit(): agg[n] = agg.get(n, 0) + int(r[i])
print("total samples", tot, "by reason:", sorted(((v, k) for k, v in agg.items()), reverse=True)[:8])
top = sorted(data, key=lambda r: -int(r[si]) if r[si].isdigit() else 0)[:int(sys.argv[2]) if len(sys.argv) > 2 else 40]
for r in top:
    rs = sorted(((int(r[i]), n[6:]) for i, n in reasons if r[i].isdigit() and int(r[i]) > 0), reverse=True)[:3]
    print(f"{r[si]:>6} {r[ex]:>8} {r[0][-5:]} {r[1][:70]:70s} {rs}")
