"""Summary of an ncu launch list (gpu__time_duration.sum per kernel): launches and time per kernel name,
share of the serialised total.    python scripts/launch_summary.py L.csv > profiles/rN_launches_C5.txt"""
import csv, io, sys
rows = [l for l in open(sys.argv[1]) if not l.startswith("==")]
by = {}
for x in csv.DictReader(io.StringIO("".join(rows))):
    d = by.setdefault(int(x["ID"]), {"k": x["Kernel Name"]})
    d[x["Metric Name"]] = float(x["Metric Value"].replace(",", ""))
agg = {}
for d in by.values():
    name = d["k"].split("(")[0].split("<")[0]
    a = agg.setdefault(name, [0, 0.0])
    a[0] += 1
    a[1] += d.get("gpu__time_duration.sum", 0.0)
tot = sum(v[1] for v in agg.values())
print(f"{len(by)} launches, {tot / 1e6:.3f} ms total (serialised, cold-cache)")
for k, (n, t) in sorted(agg.items(), key=lambda kv: -kv[1][1]):
    print(f"  {k:40s} n={n:5d} {t / 1e6:10.3f} ms {100 * t / tot:6.1f}%")
