"""Factorization time of a config under relaxed-amalgamation thresholds
(nrelax, zrelax; SURVEY Appendix B defaults {4,16,48}, {0.8,0.1,0.05}):
coarser supernodes mean fewer, larger fronts (less latency, more padding flops).
    python tools/amalg_sweep.py c2"""
import sys

sys.path.insert(0, ".")
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_ipps_georgesgsc11_b200 as mf  # noqa: E402
from workloads import grids as G  # noqa: E402

name = sys.argv[1] if len(sys.argv) > 1 else "c2"
c = G.CONFIGS[name]
A, p = G.make_config(c["kind"], c["N"])
vals = torch.from_numpy(A.values).cuda()
for nr, zr in [((4, 16, 48), (0.8, 0.1, 0.05)), ((8, 32, 96), (0.8, 0.1, 0.05)), ((8, 32, 96), (0.8, 0.2, 0.1)),
               ((16, 64, 192), (0.8, 0.2, 0.1)), ((16, 64, 192), (0.9, 0.3, 0.15))]:
    S = mf.Solver(nrelax=nr, zrelax=zr)
    S.analyze(A.n, A.colptr, A.rowind, p)
    for _ in range(3):
        S.factor(vals)
    ts = []
    for _ in range(5):
        S.factor(vals)
        ts.append(S.info()["t_factor"] * 1e3)
    inf = S.info()
    print(f"{name} nrelax={nr} zrelax={zr}: {np.median(ts):.3f} ms nsuper={inf['nsuper']} levels={inf['nlevels']} "
          f"exec/true flops={inf['flops_exec'] / inf['flops_true']:.3f} GF/s(true)={inf['flops_true'] / np.median(ts) / 1e6:.0f}",
          flush=True)
    S.close()
    torch.cuda.empty_cache()
