"""One warm c5 factorization inside a cudaProfilerStart/Stop window, for ncu
(`--profile-from-start off`).  Not a benchmark: numbers printed here are not
bench values."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_ipps_georgesgsc11_b200 as mf  # noqa: E402
from workloads import grids as G  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "c5"
c = G.CONFIGS[cfg]
A, p = G.make_config(c["kind"], c["N"])
S = mf.Solver(nbranch=int(os.environ.get("NB", "4")))
S.analyze(A.n, A.colptr, A.rowind, p)
v = torch.from_numpy(A.values).cuda()
S.factor(v)
torch.cuda.synchronize()
torch.cuda.profiler.start()
S.factor(v)
torch.cuda.synchronize()
torch.cuda.profiler.stop()
print("launches per factor:", S.info()["launches_factor"], "t_factor", S.info()["t_factor"])
