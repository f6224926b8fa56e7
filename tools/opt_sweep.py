"""Factorization time of one config under option combinations (mf_options):
python tools/opt_sweep.py c2 'nbranch=4' 'nbranch=8' 'nbranch=16,lookahead=1'"""
import sys

sys.path.insert(0, ".")
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_ipps_georgesgsc11_b200 as mf  # noqa: E402
from workloads import grids as G  # noqa: E402

name = sys.argv[1]
c = G.CONFIGS[name]
A, p = G.make_config(c["kind"], c["N"])
vals = torch.from_numpy(A.values).cuda()
for spec in sys.argv[2:] or [""]:
    kw = {}
    for item in filter(None, spec.split(",")):
        k, v = item.split("=")
        kw[k] = int(v)
    S = mf.Solver(**kw)
    S.analyze(A.n, A.colptr, A.rowind, p)
    for _ in range(3):
        S.factor(vals)
    ts = []
    for _ in range(7):
        S.factor(vals)
        ts.append(S.info()["t_factor"] * 1e3)
    print(f"{name} {spec or 'default'}: {np.median(ts):.3f} ms (min {min(ts):.3f}) launches {S.info()['launches_factor']}",
          flush=True)
    S.close()
    torch.cuda.empty_cache()
