"""Per-F-U-call trace of one factorization, in the spirit of the paper's records of
every factor-update call with its (m, k) and time [PAPER.md L95]: one profiled
factorization (CUDA events around every launch), each launch's time attributed to
the fronts of its level and kernel class in proportion to their flops (a launch
batches many fronts, so per-front times are estimates; per-launch times are exact).

    python tools/fu_trace.py c3 gpurun_out/fu_trace_c3.csv      (GPU)
columns: supernode, level, m, k, variant, est_ms, launch_share"""
import collections
import csv
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_ipps_georgesgsc11_b200 as mf  # noqa: E402
from workloads import grids as G  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "c3"
out = sys.argv[2] if len(sys.argv) > 2 else f"gpurun_out/fu_trace_{cfg}.csv"
c = G.CONFIGS[cfg]
A, p = G.make_config(c["kind"], c["N"])
S = mf.Solver(nbranch=1)
S.analyze(A.n, A.colptr, A.rowind, p)
v = torch.from_numpy(A.values).cuda()
S.factor(v)
S.set_profiling(True)
S.factor(v)
prog, times = S.program(), S.launch_times()
S.set_profiling(False)
sn = S.supernodes()
k = np.diff(sn["sn_first"]).astype(np.int64)
f = np.diff(sn["sn_rowptr"]).astype(np.int64)
m = f - k
variant = S.variants()
parent = sn["sn_parent"]
ns = len(k)
level = np.zeros(ns, dtype=np.int64)   # height in the supernodal tree (the schedule's levels)
for s in range(ns):
    if parent[s] >= 0:
        level[parent[s]] = max(level[parent[s]], level[s] + 1)
fl = k * m * m + m * k * (k + 1) + k * (k + 1) * (2 * k + 1) // 6
# launch time per (level, tiled?) -> fronts of that level and path, by flops
small_cls = {0}
t_level = collections.defaultdict(float)
for L, t in zip(prog, times):
    t_level[(L["level"], L["kind"] in small_cls)] += float(t)
est = np.zeros(ns)
share = np.zeros(ns)
for (lv, small), t in t_level.items():
    sel = np.nonzero((level == lv) & ((variant < 6) == small))[0]
    if sel.size == 0:
        continue
    w = fl[sel] / max(fl[sel].sum(), 1)
    est[sel] = t * w
    share[sel] = w
os.makedirs(os.path.dirname(out) or ".", exist_ok=True)
with open(out, "w", newline="") as fh:
    wr = csv.writer(fh)
    wr.writerow(["supernode", "level", "m", "k", "variant", "est_ms", "launch_share"])
    for s in range(ns):
        wr.writerow([s, int(level[s]), int(m[s]), int(k[s]), int(variant[s]), f"{est[s]:.6f}", f"{share[s]:.4f}"])
print(f"{cfg}: {ns} F-U calls, {len(prog)} launches, profiled {sum(times):.2f} ms -> {out}")
