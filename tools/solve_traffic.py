"""Per-kernel DRAM bytes and GB/s of one profiled solve (tools/gpu/job_solve_ncu.sh)."""
import collections
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
hi = [i for i, r in enumerate(rows) if "Kernel Name" in r][0]
h = rows[hi]
idx = {n: h.index(n) for n in ("ID", "Kernel Name", "Metric Name", "Metric Unit", "Metric Value")}
scale = {"ns": 1e-9, "nsecond": 1e-9, "usecond": 1e-6, "us": 1e-6, "msecond": 1e-3, "ms": 1e-3,
         "byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}
per = collections.defaultdict(dict)
for r in rows[hi + 1:]:
    if len(r) < len(h):
        continue
    v = float(r[idx["Metric Value"]].replace(",", "")) * scale.get(r[idx["Metric Unit"]], 1.0)
    per[r[idx["ID"]]]["name"] = r[idx["Kernel Name"]].split("(")[0].split("<")[0].replace("void ", "")
    per[r[idx["ID"]]][r[idx["Metric Name"]]] = v
agg = collections.defaultdict(lambda: [0, 0.0, 0.0])
for d in per.values():
    a = agg[d["name"]]
    a[0] += 1
    a[1] += d.get("gpu__time_duration.sum", 0.0)
    a[2] += d.get("dram__bytes_read.sum", 0.0) + d.get("dram__bytes_write.sum", 0.0)
T = sum(a[1] for a in agg.values())
B = sum(a[2] for a in agg.values())
print(f"{'kernel':16s} {'launches':>8s} {'ms':>8s} {'GB':>7s} {'GB/s':>7s}")
for n, (c, t, b) in sorted(agg.items(), key=lambda x: -x[1][1]):
    print(f"{n:16s} {c:8d} {t * 1e3:8.3f} {b / 1e9:7.3f} {b / t / 1e9:7.0f}")
print(f"{'total':16s} {len(per):8d} {T * 1e3:8.3f} {B / 1e9:7.3f} {B / T / 1e9:7.0f}")
