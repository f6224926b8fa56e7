"""Join a factor launch list (ncu --metrics gpu__time_duration.sum --csv, one
mf_factor) with the static program (host-only analyze): per-launch achieved rates."""
import csv, sys, os, collections
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import paper_conf_ipps_georgesgsc11_b200 as mf
from workloads import grids as G

path, cfg = sys.argv[1], (sys.argv[2] if len(sys.argv) > 2 else "c5")
rows = list(csv.reader(open(path)))
h = None; seq = []
scale = {"nsecond": 1e-3, "ns": 1e-3, "usecond": 1.0, "us": 1.0, "msecond": 1e3, "ms": 1e3}
for r in rows:
    if "Kernel Name" in r: h = r; continue
    if h is None or len(r) != len(h): continue
    d = dict(zip(h, r))
    if d["Metric Name"] != "gpu__time_duration.sum": continue
    seq.append((d["Kernel Name"].split("(")[0], float(d["Metric Value"].replace(",", "")) * scale.get(d["Metric Unit"], 1.0), d["Grid Size"]))
c = G.CONFIGS[cfg]
A, p = G.make_config(c["kind"], c["N"])
S = mf.Solver(host_only=True)
S.analyze(A.n, A.colptr, A.rowind, p)
prog = S.program()
assert len(seq) == len(prog) + 1, (len(seq), len(prog))
seq = seq[1:]
names = {0: "small", 1: "assemble", 2: "potrf", 3: "trsm", 4: "update", 5: "leaf", 6: "panel"}
by = collections.defaultdict(lambda: [0, 0.0, 0.0])
upd = []
for (kn, us, grid), L in zip(seq, prog):
    k = names[L["kind"]]
    by[k][0] += 1; by[k][1] += us; by[k][2] += L["flops"]
    if k == "update":
        upd.append((us, L["flops"], L["count"], L["level"], grid))
tot = sum(v[1] for v in by.values())
for k, (n, us, fl) in sorted(by.items(), key=lambda x: -x[1][1]):
    print(f"{k:10s} {n:5d} {us/1e3:8.2f} ms {100*us/tot:5.1f}%  {fl/us/1e6 if us else 0:7.2f} TF/s")
print(f"total {tot/1e3:.2f} ms")
upd = np.array([(u, f, c, l) for u, f, c, l, g in upd])
rate = upd[:, 1] / upd[:, 0] / 1e6
ideal = upd[:, 1] / 33.5e6
print("update launches:", len(upd), "time", upd[:, 0].sum() / 1e3, "ms; at 33.5 TF/s:", ideal.sum() / 1e3, "ms")
# loss by tiles-per-launch bucket
for lo, hi in [(0, 148), (148, 592), (592, 2000), (2000, 10000), (10000, 1e9)]:
    m = (upd[:, 2] >= lo) & (upd[:, 2] < hi)
    if m.any():
        print(f"tiles [{lo},{hi}): n={m.sum():4d} time {upd[m,0].sum()/1e3:7.2f} ms  ideal {ideal[m].sum()/1e3:7.2f} ms  rate {upd[m,1].sum()/upd[m,0].sum()/1e6:6.2f} TF/s")
for l in sorted(set(upd[:, 3])):
    m = upd[:, 3] == l
    print(f"level {int(l):2d}: n={m.sum():4d} time {upd[m,0].sum()/1e3:7.2f} ms ideal {ideal[m].sum()/1e3:7.2f} rate {upd[m,1].sum()/upd[m,0].sum()/1e6:6.2f}")
