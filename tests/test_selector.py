"""Learned kernel-variant selector (Sec. VI, Eqs. 3-5).

CPU: the oracle (oracle/selector.py) against what the mathematics fixes --
closed form at theta = 0, a dominant class, a 1-D cost crossing -- then the
product fit (selector.py, damped Newton) against the oracle (analytic vs
numerical gradient, attained objective vs L-BFGS), and the C planner's per-front
argmax (mf_get_variants, host-only plan) against the oracle's Eq. 5 bit-exactly.
GPU: factorizations whose fronts are spread over every kernel variant (random
theta, forced classes) against the oracle factor.
"""
import numpy as np
import pytest

import oracle
from oracle import selector as OS
from tests._grids import grid

R = 7   # classes (include/mf.h MF_VARIANTS)
FMAX = (16, 32, 64, 96, 128, 160, 0)


def feas_of(m, k):
    f = m + k
    return [fm == 0 or f <= fm for fm in FMAX]


def shapes():
    out = []
    for m in (0, 4, 12, 24, 40, 70, 100, 150, 220):
        for k in (1, 3, 8, 20, 50, 90):
            out.append((m, k))
    return out


# ------------------------------------------------------------------ oracle pins
def test_oracle_theta_zero_is_mean_time():
    # theta = 0: every feasible class equally likely -> expected time = mean over feasible classes
    rng = np.random.default_rng(0)
    sh = shapes()
    X = [OS.front_features(m, k) for m, k in sh]
    F = [feas_of(m, k) for m, k in sh]
    T = rng.uniform(1, 5, size=(len(sh), R)).tolist()
    th = np.zeros((9, R)).tolist()
    want = sum(np.mean([T[i][j] for j in range(R) if F[i][j]]) for i in range(len(sh)))
    assert abs(OS.expected_time(th, X, T, F) - want) <= 1e-12 * want


def test_oracle_dominant_class_is_learned():
    sh = [(m, k) for m, k in shapes() if m + k <= 160]
    X = [OS.front_features(m, k) for m, k in sh]
    F = [feas_of(m, k) for m, k in sh]
    T = [[1.0 if j == 5 else 2.0 for j in range(R)] for _ in sh]   # cta160 always cheapest
    th, _ = OS.fit_reference(X, T, F)
    assert all(OS.predict(th, x, f) == 5 for x, f in zip(X, F))


def test_oracle_cost_crossing():
    # two feasible classes with costs linear in a = m/64 crossing at m = 64:
    # class 0 cheaper below, class 6 above (Eq. 3's minimiser splits there)
    ms = [0, 8, 16, 24, 32, 40, 48, 56, 72, 80, 88, 96, 104, 112, 120, 128]
    k = 32
    X = [OS.front_features(m, k) for m in ms]
    F = [[j in (0, 6) for j in range(R)] for _ in ms]
    T = [[(1 + m / 64) if j == 0 else (3 - m / 64) if j == 6 else 0.0 for j in range(R)] for m in ms]
    th, _ = OS.fit_reference(X, T, F)
    pred = [OS.predict(th, x, f) for x, f in zip(X, F)]
    assert pred == [0 if m < 64 else 6 for m in ms]


# ------------------------------------------------------------------ product vs oracle (CPU)
@pytest.fixture(scope="module")
def sel():
    from paper_conf_ipps_georgesgsc11_b200 import selector
    return selector


def test_features_match_oracle(sel):
    for m, k in shapes():
        np.testing.assert_array_equal(sel.features([m], [k])[0], np.array(OS.front_features(m, k)))
        assert list(sel.feasible(np.array([m]), np.array([k]))[0]) == feas_of(m, k)


def test_gradient_matches_finite_differences(sel):
    rng = np.random.default_rng(1)
    sh = shapes()[:20]
    X = np.array([OS.front_features(m, k) for m, k in sh])
    F = np.array([feas_of(m, k) for m, k in sh])
    T = rng.uniform(0.5, 3, size=(len(sh), R))
    th = rng.normal(scale=0.3, size=(9, R))
    J, G, H = sel.objective(th, X, T, F)
    assert abs(J - OS.expected_time(th.tolist(), X.tolist(), T.tolist(), F.tolist())) <= 1e-12 * J
    Gn = OS.numerical_gradient(th.tolist(), X.tolist(), T.tolist(), F.tolist())
    np.testing.assert_allclose(G, Gn, rtol=1e-5, atol=1e-8)
    # Hessian column by finite differences of the analytic gradient
    h = 1e-6
    for q, j in [(0, 0), (2, 3), (8, 6)]:
        tp, tm = th.copy(), th.copy()
        tp[q, j] += h
        tm[q, j] -= h
        col = (sel.objective(tp, X, T, F)[1] - sel.objective(tm, X, T, F)[1]).reshape(-1) / (2 * h)
        np.testing.assert_allclose(H[:, q * R + j], col, rtol=1e-4, atol=1e-6)


def test_newton_fit_reaches_reference_objective(sel):
    # synthetic per-class costs shaped like batched kernels: fixed + per-flop terms
    sh = shapes()
    m = np.array([s[0] for s in sh], float)
    k = np.array([s[1] for s in sh], float)
    fl = k * m * m + m * k * (k + 1) + k * (k + 1) * (2 * k + 1) / 6
    f = m + k
    base = np.array([0.3, 0.5, 1.0, 1.6, 2.4, 3.5, 12.0])
    rate = np.array([4.0, 3.0, 1.0, 0.8, 0.7, 0.6, 0.05]) * 1e-4
    T = base[None, :] + rate[None, :] * fl[:, None] + 1e-3 * f[:, None] ** 2 * (np.arange(R) < 6)
    X = sel.features(m, k)
    F = sel.feasible(m, k)
    th = sel.fit(X, T, F)
    scale = T[F].mean()
    J = sel.objective(th, X, T / scale, F, 1e-6)[0]
    _, Jref = OS.fit_reference(X.tolist(), T.tolist(), F.tolist())
    assert J <= Jref * (1 + 1e-6) + 1e-9
    # the fitted policy is near the per-front best (the paper's ideal hybrid P_IH)
    pred = sel.predict(th, X, F)
    best = np.where(F, T, np.inf).min(axis=1)
    assert T[np.arange(len(sh)), pred].sum() <= 1.05 * best.sum()


def _plan_variants(A, p, theta=None, force=-1):
    import paper_conf_ipps_georgesgsc11_b200 as mf
    S = mf.Solver(host_only=True)
    S.set_variant_model(theta, force)
    S.analyze(A.n, A.colptr, A.rowind, p)
    sn = S.supernodes()
    return S, S.variants(), sn


def test_planner_argmax_matches_oracle_eq5():
    A, p = grid("27pt", (14, 13, 12))
    rng = np.random.default_rng(7)
    for trial in range(3):
        th = rng.normal(size=(9, R))
        S, var, sn = _plan_variants(A, p, th)
        k = np.diff(sn["sn_first"])
        f = np.diff(sn["sn_rowptr"])
        for s in range(len(k)):
            m_s, k_s = int(f[s] - k[s]), int(k[s])
            want = OS.predict(th.tolist(), OS.front_features(m_s, k_s), feas_of(m_s, k_s))
            assert var[s] == want, (s, m_s, k_s)
        S.close()


def test_planner_force_and_default():
    from paper_conf_ipps_georgesgsc11_b200 import selector as sel
    A, p = grid("27pt", (12, 12, 12))
    S, var, sn = _plan_variants(A, p)
    k = np.diff(sn["sn_first"])
    f = np.diff(sn["sn_rowptr"])
    np.testing.assert_array_equal(var, sel.baseline_class(f - k, k))
    S.close()
    for force in range(R):
        S, var, sn = _plan_variants(A, p, None, force)
        feas = np.array([feas_of(int(f[s] - k[s]), int(k[s]))[force] for s in range(len(k))])
        assert (var[feas] == force).all()
        S.close()


# ------------------------------------------------------------------ GPU: every variant factors correctly
@pytest.mark.gpu
@pytest.mark.parametrize("mode", ["random0", "random1", "force_tiled", "force_cta160", "force_warp32"])
def test_gpu_variants_parity(mode):
    import torch
    assert torch.cuda.is_available()
    import paper_conf_ipps_georgesgsc11_b200 as mf
    A, p = grid("27pt", (14, 13, 12))
    S = mf.Solver()
    if mode.startswith("random"):
        S.set_variant_model(np.random.default_rng(int(mode[-1])).normal(size=(9, R)))
    else:
        S.set_variant_model(None, {"force_tiled": 6, "force_cta160": 5, "force_warp32": 1}[mode])
    S.analyze(A.n, A.colptr, A.rowind, p)
    used = set(S.variants().tolist())
    S.factor(A.values)
    sym = oracle.symbolic(A, p)
    panels = oracle.factor(A, sym)
    worst = 0.0
    for s, Po in panels.items():
        fr, kk = Po.shape
        Pg = S.panel(s, fr, kk)
        colmax = np.abs(Po).max(axis=0)
        den = np.maximum(np.abs(Po), 1e-6 * colmax[None, :])
        den[den == 0] = 1.0
        worst = max(worst, float((np.abs(Pg - Po) / den).max()))
    assert worst <= 1e-10, (mode, worst, used)
    if mode.startswith("random"):
        assert len(used) >= 2, used


def test_packaged_model_is_the_default_and_feasible():
    """The fitted selector shipped with the binding (variant_model.json, fitted by
    tools/fit_variant_model.py --relative on B200 timings) is loaded by default and
    every class it picks can run its front (order bound >= f)."""
    import paper_conf_ipps_georgesgsc11_b200 as mf
    from paper_conf_ipps_georgesgsc11_b200 import selector as sel
    th = sel.load_model()
    assert th is not None and th.shape == (9, R)
    A, p = grid("27pt", (12, 12, 12))
    S = mf.Solver(host_only=True)
    assert S.variant_model == sel.MODEL_PATH
    S.analyze(A.n, A.colptr, A.rowind, p)
    sn = S.supernodes()
    k = np.diff(sn["sn_first"])
    f = np.diff(sn["sn_rowptr"])
    var = S.variants()
    feas = sel.feasible(f - k, k)
    assert feas[np.arange(len(var)), var].all()
    # Eq. 5 over the feasible classes, as the planner evaluates it
    np.testing.assert_array_equal(var, sel.predict(th, sel.features(f - k, k), feas))
    S.close()
    S = mf.Solver(host_only=True, variant_model=None)
    S.analyze(A.n, A.colptr, A.rowind, p)
    np.testing.assert_array_equal(S.variants(), sel.baseline_class(f - k, k))
    S.close()
