"""Per-level, per-kernel-class time of one profiled factorization (CUDA events
around every launch, serialised): where the step goes, and at what rate.

    python tools/level_breakdown.py [c5] [nbranch]        (GPU)
Not a benchmark: the profiled replay serialises the launches."""
import collections
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_ipps_georgesgsc11_b200 as mf  # noqa: E402
from workloads import grids as G  # noqa: E402

NAMES = {0: "small", 1: "assemble", 2: "potrf", 3: "trsm", 4: "update", 5: "leaf", 6: "panel", 16: "xchg"}


def main():
    cfg = sys.argv[1] if len(sys.argv) > 1 else "c5"
    nb = int(sys.argv[2]) if len(sys.argv) > 2 else 1
    c = G.CONFIGS[cfg]
    A, p = G.make_config(c["kind"], c["N"])
    S = mf.Solver(nbranch=nb)
    S.analyze(A.n, A.colptr, A.rowind, p)
    v = torch.from_numpy(A.values).cuda()
    S.factor(v)
    prog = S.program()
    best = None
    for _ in range(3):
        S.set_profiling(True)
        S.factor(v)
        t = S.launch_times()
        best = t if best is None or t.sum() < best.sum() else best
    t = best
    print(f"{cfg}: {len(prog)} launches, profiled sum {t.sum():.2f} ms")
    by = collections.defaultdict(lambda: [0, 0.0, 0.0, 0.0])
    for L, ms in zip(prog, t):
        k = (L["level"], NAMES.get(L["kind"], str(L["kind"])))
        e = by[k]
        e[0] += 1; e[1] += ms; e[2] += L["flops"]; e[3] += L["bytes"]
    levels = sorted({k[0] for k in by})
    tot = collections.defaultdict(float)
    for l in levels:
        parts = []
        for (ll, name), (n, ms, fl, b) in sorted(by.items()):
            if ll != l:
                continue
            tot[name] += ms
            rate = f"{fl / ms / 1e9:6.2f}TF" if fl else f"{b / ms / 1e6:6.0f}GB/s"
            parts.append(f"{name}:{n}x {ms:7.2f}ms {rate}")
        print(f"L{l:2d} " + " | ".join(parts))
    print("totals:", {k: round(v, 2) for k, v in tot.items()})
    if os.environ.get("DUMP"):
        import json
        json.dump([dict(L, ms=float(ms)) for L, ms in zip(prog, t)], open(os.environ["DUMP"], "w"))
    sn = S.supernodes()
    first, par = sn["sn_first"], sn["sn_parent"]
    k = np.diff(first)
    f = np.diff(sn["sn_rowptr"])
    order = np.argsort(-f)[:12]
    print("largest fronts (s, k, f, parent):", [(int(s), int(k[s]), int(f[s]), int(par[s])) for s in order])


if __name__ == "__main__":
    main()
