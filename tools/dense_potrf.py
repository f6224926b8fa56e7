"""Dense POTRF calibration on the paper's root-front shapes (Table V, P:L353-377:
m = 0 root fronts, k = 5418 / 10592 / 5353 / 5682 / 7014; plus c5's root 14900).

A dense SPD matrix is one supernode, so mf_factor runs exactly the large-front
path of a root front (assembly + recursive blocked potrf).  cuSOLVER's dpotrf
(torch.linalg.cholesky) on the same matrix is printed next to it as a library
calibration.  Wall-clock around synchronised calls; not a bench value.
"""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_ipps_georgesgsc11_b200 as mf  # noqa: E402

PROF = "--prof" in sys.argv   # one extra factorization inside cudaProfilerStart/Stop (ncu --profile-from-start off)
ks = [int(x) for x in sys.argv[1:] if x != "--prof"] or [5418, 10592, 5353, 5682, 7014, 14900]
for k in ks:
    rng = np.random.default_rng(k)
    # lower CSC of A = B + k I, B symmetric uniform(-1, 1): SPD by diagonal dominance
    colptr = np.zeros(k + 1, np.int64)
    colptr[1:] = np.cumsum(np.arange(k, 0, -1))
    rowind = np.concatenate([np.arange(j, k, dtype=np.int32) for j in range(k)])
    vals = rng.uniform(-1, 1, size=rowind.size)
    vals[colptr[:-1]] = 2.0 * k
    S = mf.Solver(lookahead=bool(int(os.environ.get("MF_LA", "0"))))   # MF_LA=1: look-ahead schedule
    S.analyze(k, colptr, rowind, np.arange(k, dtype=np.int32))
    v = torch.from_numpy(vals).cuda()
    S.factor(v)
    torch.cuda.synchronize()
    ts = []
    for _ in range(5):
        t0 = time.perf_counter()
        S.factor(v)
        torch.cuda.synchronize()
        ts.append(time.perf_counter() - t0)
    t = min(ts)
    if PROF:
        torch.cuda.profiler.start()
        S.factor(v)
        torch.cuda.synchronize()
        torch.cuda.profiler.stop()
    fl = sum((i * i) for i in range(1, k + 1))
    # cuSOLVER on the dense matrix
    D = torch.zeros(k, k, dtype=torch.float64, device="cuda")
    cols = torch.from_numpy(np.repeat(np.arange(k), np.diff(colptr))).cuda()
    rows = torch.from_numpy(rowind.astype(np.int64)).cuda()
    D[rows, cols] = v
    D = D + D.tril(-1).T
    torch.linalg.cholesky(D)
    torch.cuda.synchronize()
    tc = []
    for _ in range(5):
        t0 = time.perf_counter()
        torch.linalg.cholesky(D)
        torch.cuda.synchronize()
        tc.append(time.perf_counter() - t0)
    print(f"k={k:6d}  mf {t*1e3:8.2f} ms {fl/t/1e12:6.2f} TF/s   cusolver {min(tc)*1e3:8.2f} ms {fl/min(tc)/1e12:6.2f} TF/s "
          f"launches {S.info()['launches_factor']}", flush=True)
    S.close()
    del D, v
