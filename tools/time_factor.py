"""Time mf_factor on a config (CUDA events, graph replay, device-resident values):
    [MF_*=...] python tools/time_factor.py c3 [c5 ...]      (GPU; one line per config)
Used for A/B runs of environment-selected variants (each setting in its own process:
the planner reads MF_* once)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_ipps_georgesgsc11_b200 as mf  # noqa: E402
from workloads import grids as G  # noqa: E402

tag = " ".join(f"{k}={v}" for k, v in sorted(os.environ.items()) if k.startswith("MF_"))
for cfg in sys.argv[1:]:
    c = G.CONFIGS[cfg]
    A, p = G.make_config(c["kind"], c["N"])
    v = torch.from_numpy(A.values).cuda()
    S = mf.Solver()
    S.analyze(A.n, A.colptr, A.rowind, p)
    for _ in range(3):
        S.factor(v)
    torch.cuda.synchronize()
    ts = []
    for _ in range(7):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        S.factor(v)
        e1.record()
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1))
    ts.sort()
    print(f"{cfg} [{tag}]: min {ts[0]:.3f} ms  median {ts[3]:.3f} ms  launches {S.info()['launches_factor']}",
          flush=True)
    S.close()
