"""Summarise an ncu --metrics gpu__time_duration.sum launch list (csv) for profiles/:
per kernel: launches, total us, share."""
import collections, csv, sys
rows = [r for r in csv.reader(open(sys.argv[1])) if len(r) > 14 and r[12] == "gpu__time_duration.sum"]
agg = collections.OrderedDict()
for r in rows:
    name = r[4].split("(")[0].replace("void ", "")
    t = float(r[14].replace(",", "")) / (1e3 if r[13] == "ns" else 1.0)
    c, s = agg.get(name, (0, 0.0))
    agg[name] = (c + 1, s + t)
tot = sum(s for _, s in agg.values())
out = [f"# {sys.argv[1]}: {len(rows)} launches, {tot:.1f} us total (ncu, serialised, cold cache)",
       f"{'kernel':60s} {'launches':>8s} {'total_us':>10s} {'share':>6s}"]
for k, (c, s) in sorted(agg.items(), key=lambda kv: -kv[1][1]):
    out.append(f"{k[:60]:60s} {c:8d} {s:10.1f} {s / tot:6.3f}")
print("\n".join(out))
