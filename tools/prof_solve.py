"""One warm c5 solve inside a cudaProfilerStart/Stop window, for ncu."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import paper_conf_ipps_georgesgsc11_b200 as mf
from workloads import grids as G
cfg = sys.argv[1] if len(sys.argv) > 1 else "c5"
c = G.CONFIGS[cfg]
A, p = G.make_config(c["kind"], c["N"])
S = mf.Solver(); S.analyze(A.n, A.colptr, A.rowind, p); S.factor(A.values)
b = torch.from_numpy(G.rhs(A.n, 0)).cuda(); x = torch.empty_like(b)
S.solve(b, x); torch.cuda.synchronize()
torch.cuda.profiler.start(); S.solve(b, x); torch.cuda.synchronize(); torch.cuda.profiler.stop()
print("t_solve", S.info()["t_solve"])
