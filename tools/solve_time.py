"""Device time of mf_solve (graph replay, device b / x) and of mf_solve_nrhs on a
config, after one warm-up solve (which also runs the per-factorization solve
setup).  python tools/solve_time.py c5"""
import sys

sys.path.insert(0, ".")
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_ipps_georgesgsc11_b200 as mf  # noqa: E402
from workloads import grids as G  # noqa: E402

name = sys.argv[1] if len(sys.argv) > 1 else "c5"
c = G.CONFIGS[name]
A, p = G.make_config(c["kind"], c["N"])
S = mf.Solver()
S.analyze(A.n, A.colptr, A.rowind, p)
S.factor(torch.from_numpy(A.values).cuda())
b = torch.from_numpy(G.rhs(A.n, 0)).cuda()
x = torch.empty_like(b)
S.solve(b, x)
t_first = S.info()["t_solve"]
ts = []
for _ in range(5):
    S.solve(b, x)
    ts.append(S.info()["t_solve"] * 1e3)
B = torch.from_numpy(np.random.default_rng(1).uniform(-1, 1, (8, A.n))).cuda()
S.solve_nrhs(B)
tn = S.info()["t_solve"] * 1e3
bh = G.rhs(A.n, 0)
S.solve(bh)
th = S.info()["t_solve"] * 1e3
stored = S.info()["panel_words"] * 8
print(f"{name}: solve {np.median(ts):.3f} ms (first, incl. setup {t_first * 1e3:.3f} ms; host b/x {th:.3f} ms); "
      f"nrhs=8 {tn:.3f} ms ({tn / 8:.3f} per rhs); HBM bound 2 x {stored / 1e9:.2f} GB / 6.46 TB/s = "
      f"{2 * stored / 6.46e12 * 1e3:.3f} ms")
