"""A/B timing of a factorization option (CUDA events around mf_factor, graph
replay, device-resident values):  python tools/la_ab.py c5 lookahead=0,1 [nbranch=4]"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_ipps_georgesgsc11_b200 as mf
from workloads import grids as G

cfg = sys.argv[1]
opt, vals = sys.argv[2].split("=")
extra = dict(kv.split("=") for kv in sys.argv[3:])
c = G.CONFIGS[cfg]
A, p = G.make_config(c["kind"], c["N"])
v = torch.from_numpy(A.values).cuda()
for val in vals.split(","):
    kw = {opt: int(val)}
    kw.update({k: int(x) for k, x in extra.items()})
    model = kw.pop("model", 0)     # model=1: the fitted variant selector (selector.load_model)
    S = mf.Solver(**kw)
    if model:
        from paper_conf_ipps_georgesgsc11_b200 import selector as sel
        S.set_variant_model(sel.load_model())
    S.analyze(A.n, A.colptr, A.rowind, p)
    for _ in range(3):
        S.factor(v)
    torch.cuda.synchronize()
    ts = []
    for _ in range(5):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(); S.factor(v); e1.record(); torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1))
    print(f"{cfg} {kw}: min {min(ts):.3f} ms  median {sorted(ts)[2]:.3f} ms  launches {S.info()['launches_factor']}",
          flush=True)
    S.close()
