"""Per-launch rate of the DMMA Schur-update launches of one profiled factorization
(CUDA events per launch, serialised replay): where the update loses against its
large-SYRK rate.  python tools/update_launches.py [c5]   (GPU)"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_ipps_georgesgsc11_b200 as mf  # noqa: E402
from workloads import grids as G  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "c5"
c = G.CONFIGS[cfg]
A, p = G.make_config(c["kind"], c["N"])
S = mf.Solver()
S.analyze(A.n, A.colptr, A.rowind, p)
v = torch.from_numpy(A.values).cuda()
S.factor(v)
S.set_profiling(True)
S.factor(v)
ms = np.array(S.launch_times())
S.set_profiling(False)
prog = S.program()
REF = 34.0e12   # large-SYRK rate of the kernel (profiles/r01s3_summary.md)
rows = []
for i, L in enumerate(prog):
    if L["kind"] != 4 or L["flops"] <= 0:
        continue
    t = ms[i] * 1e-3
    rows.append((L["level"], L["count"], L["flops"], L["bytes"], t, t - L["flops"] / REF))
rows.sort(key=lambda r: -r[5])
tot = sum(r[4] for r in rows)
lost = sum(r[5] for r in rows)
print(f"{cfg}: {len(rows)} update launches, {tot * 1e3:.2f} ms, {sum(r[2] for r in rows) / tot / 1e12:.2f} TF/s;"
      f" time above {REF / 1e12:.0f} TF/s: {lost * 1e3:.2f} ms")
print("level tiles  GFLOP   GB    ms    TF/s  lost_ms  AI(flop/B)")
for r in rows[:40]:
    print(f"{r[0]:5d} {r[1]:6d} {r[2] / 1e9:7.1f} {r[3] / 1e9:5.2f} {r[4] * 1e3:6.3f} {r[2] / r[4] / 1e12:6.2f} {r[5] * 1e3:7.3f}"
          f" {r[2] / max(r[3], 1):7.1f}")
by_level = {}
for r in rows:
    b = by_level.setdefault(r[0], [0, 0.0, 0.0, 0.0])
    b[0] += 1
    b[1] += r[2]
    b[2] += r[4]
    b[3] += r[5]
print("per level: level launches GFLOP ms TF/s lost_ms")
for lv in sorted(by_level):
    b = by_level[lv]
    print(f"{lv:5d} {b[0]:4d} {b[1] / 1e9:8.1f} {b[2] * 1e3:7.2f} {b[1] / b[2] / 1e12:6.2f} {b[3] * 1e3:7.2f}")
