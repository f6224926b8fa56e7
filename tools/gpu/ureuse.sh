timeout 1500 python -m pytest tests -x -q -m gpu 2>&1 | tail -1
for r in 0 1; do MF_U_REUSE=$r python - <<'PY'
import os, sys, torch
sys.path.insert(0, '.')
import paper_conf_ipps_georgesgsc11_b200 as mf
from workloads import grids as G
for cfg in ['c5', 'c4', 'c3', 'c2']:
    c = G.CONFIGS[cfg]; A, p = G.make_config(c['kind'], c['N'])
    S = mf.Solver(); S.analyze(A.n, A.colptr, A.rowind, p)
    v = torch.from_numpy(A.values).cuda()
    for _ in range(3): S.factor(v)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    ts = []
    for _ in range(5):
        e0.record(); S.factor(v); e1.record(); torch.cuda.synchronize(); ts.append(e0.elapsed_time(e1))
    print('reuse', os.environ['MF_U_REUSE'], cfg, 'workspace GB %.2f' % (S.info()['workspace_bytes'] / 1e9), 'ms %.3f' % min(ts), flush=True)
    S.close()
PY
done
