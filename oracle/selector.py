"""CPU ORACLE of the learned policy classifier (Sec. VI-B).

TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).  Plain definitions, written
from the paper, sharing no code with paper_conf_ipps_georgesgsc11_b200/selector.py
or with plan.cpp:

  * front_features(m, k): the paper's feature list [m, k, m/k, m^2, mk, k^2, k^3, mk^2]
    (PAPER.md L427), after a constant 1, with m and k in units of 64 (R3).
  * expected_time(theta, X, T, feasible): Eq. 3's objective, sum_i sum_j
    p_theta(C_j|x_i) T_ij with the multinomial logistic p, by
    explicit loops; infeasible classes are outside the softmax (R3).
  * numerical_gradient: central differences of expected_time.
  * fit_reference: minimise Eq. 3 with a library optimiser (scipy L-BFGS with the
    numerical gradient) -- a check on the attained objective, not on theta.
  * predict(theta, x, feasible): Eq. 5, y = argmax_j x . theta_j, with the dot
    product summed in feature order (the order the C planner uses), so class ids
    compare bit-exactly.
"""
from __future__ import annotations

import math

import numpy as np


def front_features(m: float, k: float) -> list[float]:
    a, b = m / 64.0, k / 64.0
    return [1.0, a, b, m / k, a * a, a * b, b * b, b * b * b, a * b * b]


def class_probabilities(theta, x, feas) -> list[float]:
    d, r = len(theta), len(theta[0])
    z = []
    for j in range(r):
        s = 0.0
        for q in range(d):
            s += x[q] * theta[q][j]
        z.append(s)
    zmax = max(z[j] for j in range(r) if feas[j])
    e = [math.exp(z[j] - zmax) if feas[j] else 0.0 for j in range(r)]
    tot = sum(e)
    return [v / tot for v in e]


def expected_time(theta, X, T, feas) -> float:
    """Eq. 3: sum over fronts i and classes j of p_theta(C_j | x_i) T_ij."""
    total = 0.0
    for i in range(len(X)):
        p = class_probabilities(theta, X[i], feas[i])
        for j in range(len(p)):
            if feas[i][j]:
                total += p[j] * T[i][j]
    return total


def numerical_gradient(theta, X, T, feas, h: float = 1e-6) -> np.ndarray:
    th = np.array(theta, dtype=np.float64)
    g = np.zeros_like(th)
    for q in range(th.shape[0]):
        for j in range(th.shape[1]):
            tp, tm = th.copy(), th.copy()
            tp[q, j] += h
            tm[q, j] -= h
            g[q, j] = (expected_time(tp, X, T, feas) - expected_time(tm, X, T, feas)) / (2 * h)
    return g


def fit_reference(X, T, feas, reg: float = 1e-6, restarts: int = 1) -> tuple[np.ndarray, float]:
    """Minimise Eq. 3 (+ reg/2 |theta|^2, T scaled to unit mean) with scipy L-BFGS."""
    from scipy.optimize import minimize

    X = [list(map(float, x)) for x in X]
    Tn = np.array(T, dtype=np.float64)
    scale = float(Tn[np.array(feas)].mean())
    Ts = (np.where(np.array(feas), Tn, 0.0) / scale).tolist()
    d, r = len(X[0]), len(T[0])

    def f(v):
        th = v.reshape(d, r)
        return expected_time(th, X, Ts, feas) + 0.5 * reg * float((v * v).sum())

    def g(v):
        th = v.reshape(d, r)
        return numerical_gradient(th, X, Ts, feas).reshape(-1) + reg * v

    best = None
    for s in range(restarts):
        v0 = np.zeros(d * r) if s == 0 else np.random.default_rng(s).normal(scale=0.1, size=d * r)
        res = minimize(f, v0, jac=g, method="L-BFGS-B", options={"maxiter": 2000, "gtol": 1e-10})
        if best is None or res.fun < best.fun:
            best = res
    return best.x.reshape(d, r), float(best.fun)


def predict(theta, x, feas) -> int:
    """Eq. 5 over the feasible classes; ties go to the lowest class index."""
    best, arg = -math.inf, -1
    for j in range(len(theta[0])):
        if not feas[j]:
            continue
        s = 0.0
        for q in range(len(x)):
            s += x[q] * theta[q][j]
        if s > best:
            best, arg = s, j
    return arg
