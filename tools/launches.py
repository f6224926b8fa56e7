"""Summarise an ncu --metrics gpu__time_duration.sum --csv launch list by kernel."""
import csv, collections, sys
rows = list(csv.reader(open(sys.argv[1])))
h = None; agg = collections.defaultdict(lambda: [0, 0.0]); seq = []
scale = {"nsecond": 1e-3, "ns": 1e-3, "usecond": 1.0, "us": 1.0, "msecond": 1e3, "ms": 1e3}
for r in rows:
    if "Kernel Name" in r: h = r; continue
    if h is None or len(r) != len(h): continue
    d = dict(zip(h, r))
    if d["Metric Name"] != "gpu__time_duration.sum": continue
    us = float(d["Metric Value"].replace(",", "")) * scale.get(d["Metric Unit"], 1.0)
    n = d["Kernel Name"].split("(")[0].split("<")[0].replace("void ", "").replace("mf::", "")
    agg[n][0] += 1; agg[n][1] += us; seq.append((n, us))
tot = sum(v[1] for v in agg.values())
for k, (c, t) in sorted(agg.items(), key=lambda x: -x[1][1]):
    print(f"{k:32s} {c:6d} {t/1e3:9.3f} ms {100*t/tot:5.1f}%")
print(f"{'total':32s} {len(seq):6d} {tot/1e3:9.3f} ms")
print("top launches:", [(n, round(u, 1)) for n, u in sorted(seq, key=lambda x: -x[1])[:int(sys.argv[2]) if len(sys.argv) > 2 else 8]])
