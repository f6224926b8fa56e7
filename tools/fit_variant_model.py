"""Fit the kernel-variant selector (Eq. 3, Newton-Raphson) to measured
per-front variant times (tools/variant_timings.py) and compare the three
policies the paper compares (Table VII):
  P_IH  ideal hybrid: the fastest measured variant of every shape,
  P_MH  model hybrid: argmax_j x . theta_j (Eq. 5) of the fitted model,
  P_BH  baseline hybrid: the fixed front-order thresholds (plan.cpp default).

    python tools/fit_variant_model.py timings.json [--relative | --workload c2,c3,c4,c5 [--warm]] [--save [path]]

--workload: the paper's own objective (Eq. 3 over the OBSERVED F-U calls, absolute
times): every front of the named BASELINE configs whose
order a batched variant can take is an example (its nearest timed shape's
per-variant times, absolute microseconds), so each shape counts as often as the
workloads factor it -- instead of --relative (reading R5: one example per grid
shape, each normalized by its fastest variant).
"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402

from paper_conf_ipps_georgesgsc11_b200 import selector as sel  # noqa: E402


def load(path):
    d = json.load(open(path))
    rows = d["rows"]
    m = np.array([r["m"] for r in rows], float)
    k = np.array([r["k"] for r in rows], float)
    T = np.array([[np.nan if t is None else t for t in r["us_per_front"]] for r in rows], float)
    return d, m, k, T


def workload_weights(m, k, configs):
    """How many fronts of the configs fall on each timed shape (nearest (m, k) in the
    grid, fronts of order <= the largest batched class; larger fronts have only the
    tiled variant and do not enter the classifier)."""
    import paper_conf_ipps_georgesgsc11_b200 as mf
    from workloads import grids as G
    w = np.zeros(len(m))
    fmax = max(f for f in sel.VARIANT_FMAX if f > 0)
    for name in configs:
        c = G.CONFIGS[name]
        A, p = G.make_config(c["kind"], c["N"])
        S = mf.Solver(host_only=True)
        S.analyze(A.n, A.colptr, A.rowind, p)
        sn = S.supernodes()
        kk = np.diff(sn["sn_first"]).astype(float)
        mm = np.diff(sn["sn_rowptr"]).astype(float) - kk
        sel_ = (mm + kk) <= fmax
        for mi, ki in zip(mm[sel_], kk[sel_]):
            # nearest timed shape with the same feasibility (its order must not exceed f's class)
            d = (m - mi) ** 2 / 64.0 + (k - ki) ** 2
            d = np.where(m + k >= mi + ki, d, d + 1e9)   # prefer shapes no smaller than the front
            w[int(np.argmin(d))] += 1
        S.close()
    return w


def main():
    path = sys.argv[1]
    d, m, k, T = load(path)
    X = sel.features(m, k)
    F = sel.feasible(m, k) & np.isfinite(T)
    weights = np.ones(len(m))
    if "--workload" in sys.argv:
        weights = workload_weights(m, k, sys.argv[sys.argv.index("--workload") + 1].split(","))
        print("observed F-U calls mapped to timed shapes:", int(weights.sum()), "of", len(m), "shapes used:",
              int((weights > 0).sum()))
    # --relative: each shape's times divided by its fastest variant (R5): the
    # grid is not a workload sample, and in absolute time the cheap shapes (175k tiny
    # fronts in c2) would not count at all
    Tfit = T / np.nanmin(np.where(F, T, np.nan), axis=1, keepdims=True) if "--relative" in sys.argv else T
    Tfit = Tfit * weights[:, None]   # Eq. 3 is linear in T: a shape seen w times counts w times
    keep = weights > 0
    # --warm: start Newton from the saved model (Eq. 3 is not convex in theta; a cold start
    # on the workload-weighted objective stops in a worse stationary point, R5)
    th0 = sel.load_model() if "--warm" in sys.argv else None
    th = sel.fit(X[keep], np.where(F, Tfit, 0.0)[keep], F[keep], reg=1e-6, theta0=th0, verbose=False)
    pm = sel.predict(th, X, F)
    pb = sel.baseline_class(m, k)
    pi = np.where(F, T, np.inf).argmin(axis=1)
    idx = np.arange(len(m))
    tot = {"P_IH": float(T[idx, pi].sum()), "P_MH": float(T[idx, pm].sum()), "P_BH": float(T[idx, pb].sum())}
    agree = {"P_MH==P_IH": float((pm == pi).mean()), "P_BH==P_IH": float((pb == pi).mean())}
    print("sum over shapes of us/front:", {k2: round(v, 3) for k2, v in tot.items()}, agree)
    for i in range(len(m)):
        print(f"m={int(m[i]):4d} k={int(k[i]):4d}  ideal {sel.VARIANT_NAMES[pi[i]]:7s} model {sel.VARIANT_NAMES[pm[i]]:7s} "
              f"base {sel.VARIANT_NAMES[pb[i]]:7s}  T=" + " ".join("   -   " if not np.isfinite(t) else f"{t:7.3f}"
                                                            for t in T[i]))
    if "--workload" in sys.argv:   # the workloads' expected time under each policy (weighted sum)
        wt = {"P_IH": float((T[idx, pi] * weights).sum()), "P_MH": float((T[idx, pm] * weights).sum()),
              "P_BH": float((T[idx, pb] * weights).sum())}
        print("workload-weighted us (sum over observed F-U calls):", {k2: round(v, 1) for k2, v in wt.items()})
    if "--save" in sys.argv:
        i = sys.argv.index("--save")
        dst = sys.argv[i + 1] if i + 1 < len(sys.argv) and not sys.argv[i + 1].startswith("--") else sel.MODEL_PATH
        sel.save_model(th, {"fitted_on": os.path.basename(path), "gpu": d.get("gpu"),
                            "objective": ("Eq. 3, observed F-U calls of " + sys.argv[sys.argv.index("--workload") + 1]
                                          if "--workload" in sys.argv else
                                          "Eq. 3, grid shapes" + (" (relative)" if "--relative" in sys.argv else "")),
                            "training_us_sum": tot, "agreement": agree}, path=dst)
        print("saved", dst)


if __name__ == "__main__":
    main()
