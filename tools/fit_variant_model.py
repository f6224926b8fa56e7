"""Fit the kernel-variant selector (Eq. 3, Newton-Raphson) to measured
per-front variant times (tools/variant_timings.py) and compare the three
policies the paper compares (Table VII):
  P_IH  ideal hybrid: the fastest measured variant of every shape,
  P_MH  model hybrid: argmax_j x . theta_j (Eq. 5) of the fitted model,
  P_BH  baseline hybrid: the fixed front-order thresholds (plan.cpp default).

    python tools/fit_variant_model.py timings.json [--save]
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


def main():
    path = sys.argv[1]
    d, m, k, T = load(path)
    X = sel.features(m, k)
    F = sel.feasible(m, k) & np.isfinite(T)
    # --relative: each shape's times divided by its fastest variant (R5): the
    # grid is not a workload sample, and in absolute time the cheap shapes (175k tiny
    # fronts in c2) would not count at all
    Tfit = T / np.nanmin(np.where(F, T, np.nan), axis=1, keepdims=True) if "--relative" in sys.argv else T
    th = sel.fit(X, np.where(F, Tfit, 0.0), F, reg=1e-6, verbose=False)
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
    if "--save" in sys.argv:
        sel.save_model(th, {"fitted_on": os.path.basename(path), "gpu": d.get("gpu"),
                            "training_us_sum": tot, "agreement": agree})
        print("saved", sel.MODEL_PATH)


if __name__ == "__main__":
    main()
