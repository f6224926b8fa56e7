"""A/B of the Schur-update mode on a BASELINE config: FP64 DMMA vs the Ozaki
int8-tensor-core emulation (ozaki_slices).  python tools/oz_ab.py c5 0 8"""
import sys
import time

sys.path.insert(0, ".")
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_ipps_georgesgsc11_b200 as mf  # noqa: E402
from workloads import grids as G  # noqa: E402

name = sys.argv[1]
modes = [int(x) for x in sys.argv[2:]] or [0, 8]
c = G.CONFIGS[name]
A, p = G.make_config(c["kind"], c["N"])
vals = torch.from_numpy(A.values).cuda()
for oz in modes:
    S = mf.Solver(ozaki_slices=oz)
    S.analyze(A.n, A.colptr, A.rowind, p)
    for _ in range(2):
        S.factor(vals)
    ts = []
    for _ in range(5):
        S.factor(vals)
        ts.append(S.info()["t_factor"] * 1e3)
    inf = S.info()
    S.set_profiling(True)
    S.factor(vals)
    st = S.kernel_stats()
    S.set_profiling(False)
    ks = " ".join(f"{k['name']}={k['ms']:.1f}" for k in st if k["ms"] > 0)
    print(f"{name} ozaki={oz}: {np.median(ts):.2f} ms ({inf['flops_true'] / np.median(ts) / 1e9:.0f} GF/s) "
          f"oz_launches={inf['launches_ozaki']} ws={inf['workspace_bytes'] / 1e9:.1f} GB | {ks}", flush=True)
    del S
    torch.cuda.empty_cache()
