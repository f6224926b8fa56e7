"""Learned kernel-variant selector: the paper's cost-sensitive multinomial
logistic policy classifier (Sec. VI-A/B, L407-437, Eqs. 3-5),
retargeted from CPU/GPU policies to the GPU kernel variants of a front
(include/mf.h mf_set_variant_model).

    theta* = argmin_theta  sum_i sum_j p_theta(C_j | x_i) T_ij          (Eq. 3)
    p_theta(C_j | x) = exp(x . theta_j) / sum_l exp(x . theta_l)
    y(x) = argmax_j x . theta_j                                         (Eq. 5)

x_i are the features of front i (m off-diagonal rows, k pivot columns), T_ij the
measured time of front i under variant j (tools/variant_timings.py on the
B200).  The fit is the paper's Newton-Raphson, damped (Levenberg-Marquardt) and
with a line search because the expected-cost objective is not convex in
general; a small ridge term fixes the softmax's shift invariance.

Readings (R3): a constant feature is prepended to the paper's eight;
m and k are measured in units of 64; a variant that cannot run a front (its
kernel's order bound is below f) is left out of that front's softmax and
argmax.  This module is host-side training / marshalling; the per-front argmax
that the factorization uses runs inside libmf (plan.cpp), fed with theta.
"""
from __future__ import annotations

import json
import os

import numpy as np

from .mf import MF_VARIANTS, MF_VARIANT_FEATURES

# order bound of each class's kernel (0 = any order: the tiled path); mirrors
# kVariantFmax in csrc/mf_plan.h
VARIANT_FMAX = (16, 32, 64, 96, 128, 160, 0)
VARIANT_NAMES = ("warp16", "warp32", "cta64", "cta96", "cta128", "cta160", "tiled")
MODEL_PATH = os.path.join(os.path.dirname(os.path.abspath(__file__)), "variant_model.json")


def features(m, k) -> np.ndarray:
    """x(m, k) (n x 9), the same arithmetic as variant_features() in mf_plan.h."""
    m = np.asarray(m, dtype=np.float64)
    k = np.asarray(k, dtype=np.float64)
    a, b = m / 64.0, k / 64.0
    return np.stack([np.ones_like(a), a, b, m / k, a * a, a * b, b * b, b * b * b, a * b * b], axis=-1)


def feasible(m, k) -> np.ndarray:
    """n x r boolean: class j can factor a front of order f = m + k."""
    f = np.asarray(m) + np.asarray(k)
    fm = np.array(VARIANT_FMAX)
    return (fm[None, :] == 0) | (f[:, None] <= fm[None, :])


def _probs(Z: np.ndarray, mask: np.ndarray) -> np.ndarray:
    Z = np.where(mask, Z, -np.inf)
    Z = Z - Z.max(axis=1, keepdims=True)
    E = np.where(mask, np.exp(Z), 0.0)
    return E / E.sum(axis=1, keepdims=True)


def objective(theta: np.ndarray, X: np.ndarray, T: np.ndarray, mask: np.ndarray, reg: float = 0.0):
    """Expected time sum_i sum_j p_ij T_ij (+ reg/2 |theta|^2), its gradient and Hessian
    (d*r square, theta flattened row-major: index q * r + j)."""
    n, d = X.shape
    r = T.shape[1]
    P = _probs(X @ theta, mask)
    Tm = np.where(mask, T, 0.0)
    E = (P * Tm).sum(axis=1)                        # expected time per front
    J = E.sum() + 0.5 * reg * float((theta * theta).sum())
    D = P * (Tm - E[:, None])                       # dE_i / dz_il = p_il (T_il - E_i)
    G = X.T @ D + reg * theta                       # d x r
    # d2E_i / dz_il dz_im = p_il (delta_lm - p_im)(T_il - E_i) - p_il p_im (T_im - E_i)
    H = np.zeros((d, r, d, r))
    for l in range(r):
        for mm in range(r):
            w = -P[:, l] * P[:, mm] * (Tm[:, l] - E) - P[:, l] * P[:, mm] * (Tm[:, mm] - E)
            if l == mm:
                w = w + P[:, l] * (Tm[:, l] - E)
            H[:, l, :, mm] = (X * w[:, None]).T @ X
    H = H.reshape(d * r, d * r) + reg * np.eye(d * r)
    return J, G, H


def fit(X: np.ndarray, T: np.ndarray, mask: np.ndarray | None = None, reg: float = 1e-6, iters: int = 200,
        theta0: np.ndarray | None = None, verbose: bool = False) -> np.ndarray:
    """Damped Newton-Raphson on Eq. 3.  T is scaled to unit mean internally (the
    minimiser does not change) so that `reg` is dimensionless."""
    X = np.asarray(X, dtype=np.float64)
    T = np.asarray(T, dtype=np.float64)
    if mask is None:
        mask = np.isfinite(T)
    T = np.where(mask, T, 0.0)
    scale = float(T[mask].mean()) or 1.0
    Ts = T / scale
    d, r = X.shape[1], T.shape[1]
    theta = np.zeros((d, r)) if theta0 is None else np.array(theta0, dtype=np.float64)
    lam = 1e-3
    J, G, H = objective(theta, X, Ts, mask, reg)
    for it in range(iters):
        g = G.reshape(-1)
        if np.abs(g).max() < 1e-10 * max(1.0, abs(J)):
            break
        improved = False
        for _ in range(30):
            A = H + lam * np.eye(d * r)
            try:
                step = np.linalg.solve(A, -g)
            except np.linalg.LinAlgError:
                lam *= 10
                continue
            cand = theta + step.reshape(d, r)
            Jc = objective(cand, X, Ts, mask, reg)[0]
            if Jc < J:
                theta = cand
                lam = max(lam / 3, 1e-12)
                improved = True
                break
            lam *= 10
        if not improved:
            break
        Jold = J
        J, G, H = objective(theta, X, Ts, mask, reg)
        if verbose:
            print(f"newton {it}: J = {J * scale:.6g} lam = {lam:.2e}")
        if Jold - J < 1e-13 * abs(Jold):
            break
    return theta


def predict(theta: np.ndarray, X: np.ndarray, mask: np.ndarray) -> np.ndarray:
    """Eq. 5 over the feasible classes."""
    Z = np.where(mask, X @ theta, -np.inf)
    return Z.argmax(axis=1)


def baseline_class(m, k, small_max: int = 128) -> np.ndarray:
    """The default front-order thresholds of plan.cpp (the analogue of the paper's
    baseline hybrid P_BH): size classes f <= 16 / 32 / 64 / 96 /
    small_max (each capped at small_max), each run by the first variant whose
    order bound covers the class bound; larger fronts tiled."""
    f = np.asarray(m) + np.asarray(k)
    out = np.full(f.shape, len(VARIANT_FMAX) - 1)

    def cls(bound):
        return next(j for j, fm in enumerate(VARIANT_FMAX) if fm == 0 or bound <= fm)

    for bound in sorted({small_max, min(96, small_max), min(64, small_max), min(32, small_max),
                         min(16, small_max)}, reverse=True):
        out[f <= bound] = cls(bound)
    return out


def save_model(theta: np.ndarray, meta: dict, path: str = MODEL_PATH) -> None:
    with open(path, "w") as fh:
        json.dump({"theta": np.asarray(theta).tolist(), "features": MF_VARIANT_FEATURES, "classes": MF_VARIANTS,
                   "class_names": VARIANT_NAMES, **meta}, fh, indent=1)


def load_model(path: str = MODEL_PATH) -> np.ndarray | None:
    if not os.path.exists(path):
        return None
    with open(path) as fh:
        th = np.array(json.load(fh)["theta"], dtype=np.float64)
    if th.shape != (MF_VARIANT_FEATURES, MF_VARIANTS):
        raise ValueError(f"bad variant model shape {th.shape}")
    return th
