set -x
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_multigpu.py -x -q -m gpu 2>&1 | tail -5
python - <<'PY'
import sys; sys.path.insert(0,'.')
import numpy as np, torch, paper_conf_ipps_georgesgsc11_b200 as mf
from workloads import grids as G
for cfg in ["c4","c5"]:
    c=G.CONFIGS[cfg]; A,p=G.make_config(c["kind"],c["N"])
    S=mf.Solver(); S.analyze(A.n,A.colptr,A.rowind,p); S.factor(A.values)
    b=torch.from_numpy(G.rhs(A.n,0)).cuda(); x=torch.empty_like(b)
    ts=[]
    for i in range(6):
        S.solve(b,x); torch.cuda.synchronize(); ts.append(S.info()["t_solve"])
    print(cfg,"t_solve ms",[round(t*1e3,3) for t in ts])
PY
ncu --metrics gpu__time_duration.sum --clock-control none --profile-from-start off --csv --log-file gpurun_out/solve_launches.csv python tools/prof_solve.py c5 > gpurun_out/solve_prof.log 2>&1
