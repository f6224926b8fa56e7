"""Per-launch CUDA-event times of the Schur-update launches, FP64 DMMA vs Ozaki
(same program, launch by launch): python tools/oz_launches.py c5 8"""
import sys

sys.path.insert(0, ".")
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_ipps_georgesgsc11_b200 as mf  # noqa: E402
from workloads import grids as G  # noqa: E402

name, oz = sys.argv[1], int(sys.argv[2])
c = G.CONFIGS[name]
A, p = G.make_config(c["kind"], c["N"])
vals = torch.from_numpy(A.values).cuda()
res = {}
for mode in (0, oz):
    S = mf.Solver(ozaki_slices=mode)
    S.analyze(A.n, A.colptr, A.rowind, p)
    S.factor(vals)
    S.set_profiling(True)
    S.factor(vals)
    res[mode] = (S.program(), S.launch_times())
    S.set_profiling(False)
    del S
    torch.cuda.empty_cache()
prog, t0 = res[0]
_, t1 = res[oz]
rows = []
for i, L in enumerate(prog):
    if L["kind"] != 4:
        continue
    kavg = L["flops"] / (2.0 * 64 * 64 * max(L["count"], 1))
    rows.append((t0[i], t1[i], kavg, L["count"], L["flops"], L["level"]))
rows.sort(key=lambda r: -r[0])
tot0 = sum(r[0] for r in rows)
tot1 = sum(r[1] for r in rows)
print(f"{name}: update launches {len(rows)}: dmma {tot0:.1f} ms, ozaki{oz} {tot1:.1f} ms")
print(" dmma_ms  oz_ms  ratio   kavg  tiles64   TF/s(dmma) level")
for r in rows[:40]:
    print(f"{r[0]:8.3f} {r[1]:7.3f} {r[0] / max(r[1], 1e-9):6.2f} {r[2]:7.0f} {r[3]:7d} {r[4] / r[0] / 1e9:8.1f} {r[5]:3d}")
for lo, hi in [(0, 256), (256, 512), (512, 1024), (1024, 2048), (2048, 4096), (4096, 1e9)]:
    sel = [r for r in rows if lo <= r[2] < hi]
    if sel:
        print(f"K in [{lo},{hi}): n={len(sel)} dmma {sum(r[0] for r in sel):.1f} ms  oz {sum(r[1] for r in sel):.1f} ms")
