"""Measure T_ij, the per-front time of every kernel variant on a grid of front
shapes (m off-diagonal rows, k pivot columns) -- the observed timing data the
paper's policy classifier is fitted to (Sec. VI-B: "T_ij = T(A_i, C_j)
denote the observed computational time for the matrix A_i using the policy C_j").

For a shape (m, k) the matrix is B copies of [child (k) | child (k) | parent (m)]:
each child is a dense k-column supernode whose m off-diagonal rows are the
parent's columns (two children, so fundamental supernodes never merge them with
the parent; amalgamation off).  The 2B children form tree level 0; the factor
runs with the variant forced (mf_set_variant_model force = j) and profiled, and
T_ij = (sum of the level-0 launch times) / (2B).

    python tools/variant_timings.py [out.json]        (GPU)
"""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_ipps_georgesgsc11_b200 as mf  # noqa: E402
from paper_conf_ipps_georgesgsc11_b200 import selector as sel  # noqa: E402

NNZ_BUDGET = 3_000_000
M_GRID = (0, 4, 8, 16, 24, 32, 48, 64, 96, 128, 160, 224)
K_GRID = (1, 2, 4, 8, 16, 24, 32, 48, 64, 96, 128)


def forest(m: int, k: int, B: int, seed: int = 0):
    """Lower CSC of B copies of [child k | child k | parent m], SPD by diagonal dominance."""
    n1 = 2 * k + m
    cols_rows = []
    for j in range(n1):
        if j < 2 * k:
            c0 = (j // k) * k
            rows = list(range(j, c0 + k)) + list(range(2 * k, n1))
        else:
            rows = list(range(j, n1))
        cols_rows.append(rows)
    per = np.array([len(r) for r in cols_rows])
    rows1 = np.concatenate([np.array(r, dtype=np.int64) for r in cols_rows])
    n = B * n1
    colptr = np.zeros(n + 1, dtype=np.int64)
    colptr[1:] = np.cumsum(np.tile(per, B))
    rowind = (rows1[None, :] + n1 * np.arange(B)[:, None]).reshape(-1).astype(np.int32)
    rng = np.random.default_rng(seed)
    vals = rng.uniform(-0.5, 0.5, size=rowind.size)
    diag_pos = colptr[:-1]
    vals[diag_pos] = float(n1)
    return n, colptr, rowind, vals


def time_variant(m, k, B, j, vals_dev, n, colptr, rowind):
    S = mf.Solver(amalgamate=False, nbranch=1)
    S.set_variant_model(None, j)
    S.analyze(n, colptr, rowind, np.arange(n, dtype=np.int32))
    var = S.variants()
    prog = S.program()
    S.set_profiling(True)
    S.factor(vals_dev)
    best = None
    for _ in range(3):
        S.set_profiling(True)
        S.factor(vals_dev)
        t = S.launch_times()
        lv0 = sum(t[i] for i, L in enumerate(prog) if L["level"] == 0)
        best = lv0 if best is None else min(best, lv0)
    nchild = int((np.array([L["level"] for L in prog]) == 0).any())
    S.close()
    return best / (2 * B) * 1e3, var   # us per front


def main():
    out = sys.argv[1] if len(sys.argv) > 1 else "gpurun_out/variant_timings.json"
    rows = []
    t0 = time.time()
    for m in M_GRID:
        for k in K_GRID:
            f = m + k
            if f > 320:
                continue
            n1 = 2 * k + m
            nnz1 = 2 * (k * (k + 1) // 2 + k * m) + m * (m + 1) // 2
            B = int(np.clip(NNZ_BUDGET // max(nnz1, 1), 16, 2048))
            n, colptr, rowind, vals = forest(m, k, B)
            vd = torch.from_numpy(vals).cuda()
            feas = sel.feasible(np.array([m]), np.array([k]))[0]
            T = [None] * len(sel.VARIANT_FMAX)
            for j in range(len(T)):
                if not feas[j]:
                    continue
                us, var = time_variant(m, k, B, j, vd, n, colptr, rowind)
                T[j] = us
            rows.append({"m": m, "k": k, "B": B, "fronts": 2 * B, "us_per_front": T})
            print(f"m={m:4d} k={k:4d} B={B:5d} " + " ".join("-" if t is None else f"{t:8.3f}" for t in T),
                  flush=True)
    json.dump({"what": "per-front time (us) of each kernel variant, level-0 launches / fronts, profiled "
                       "(CUDA events per launch), 2B identical fronts per level",
               "classes": sel.VARIANT_NAMES, "rows": rows, "seconds": time.time() - t0,
               "gpu": torch.cuda.get_device_name(0)}, open(out, "w"), indent=1)


if __name__ == "__main__":
    main()
