"""Per-launch table of an ncu launch list (gpu__time_duration.sum) of one solve:
kernel, grid, microseconds, and the per-kernel totals.  python tools/solve_launch_table.py file.csv"""
import collections
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
hi = [i for i, r in enumerate(rows) if "Kernel Name" in r][0]
h = rows[hi]
kn, mv, un = h.index("Kernel Name"), h.index("Metric Value"), h.index("Metric Unit")
gs = h.index("Grid Size") if "Grid Size" in h else None
scale = {"ns": 1e-3, "nsecond": 1e-3, "usecond": 1.0, "us": 1.0, "msecond": 1e3, "ms": 1e3}
agg = collections.defaultdict(lambda: [0, 0.0])
tot = 0.0
for r in rows[hi + 1:]:
    if len(r) <= mv:
        continue
    v = float(r[mv].replace(",", "")) * scale.get(r[un], 1.0)
    name = r[kn].split("(")[0].split("<")[0].replace("void ", "")
    agg[name][0] += 1
    agg[name][1] += v
    tot += v
    if "-v" in sys.argv:
        print(f"{name:22s} {v:9.1f} us  grid {r[gs] if gs is not None else ''}")
for k, (c, t) in sorted(agg.items(), key=lambda x: -x[1][1]):
    print(f"{k:40s} {c:5d} {t / 1e3:8.3f} ms")
print(f"total {tot / 1e3:.3f} ms")
