"""Pins for the oracle's numeric part (oracle/numeric.py) against things other
than itself: hand-worked exact factors, the textbook
dense Cholesky (LAPACK on the dense P A P^T; a special case the sparse method
must reduce to), the 1D-Laplacian closed form, closed-form log-determinants of
the Laplacian stencils (eigenvalues of Kronecker sums), manufactured matrices
whose integer factor is known exactly, reconstruction and backward error.

The method: PAPER.md L27 (Sec. II-A) and Fig. 1 (L33-65)."""
import json
import os

import numpy as np
import pytest
import scipy.linalg
from hypothesis import given, settings, strategies as st

import oracle
from workloads import grids as G
from tests._grids import dense_from_rows, grid

GOLD = os.path.join(os.path.dirname(__file__), "golden")
U = 2.0 ** -53


def dense_L(A, sym):
    M = G.full_symmetric_dense(A)
    p = sym.perm
    return np.linalg.cholesky(M[np.ix_(p, p)]), M


def floored_rel(Lgot, Lref):
    """Reading C11: |dL| / max(|L_ref|, 1e-6 * max_i |L_ref(:, j)|)."""
    colmax = np.abs(Lref).max(axis=0)
    den = np.maximum(np.abs(Lref), 1e-6 * colmax[None, :])
    den[den == 0] = 1.0
    return float((np.abs(Lgot - Lref) / den).max())


def test_appendix_c_exact():
    ex = json.load(open(os.path.join(GOLD, "appendixC_examples.json")))
    for key in ("ex3", "ex4"):
        A = dense_from_rows(ex[key]["A"])
        sym = oracle.symbolic(A, None)
        L = oracle.panels_to_dense_L(sym, oracle.factor(A, sym))
        np.testing.assert_array_equal(L, np.array(ex[key]["L"], dtype=float))
    # fundamental trace of the 4x4 example: U_0 = -[[1],[1,1]] on rows {2,3}
    A = dense_from_rows(ex["ex4"]["A"])
    sym = oracle.symbolic(A, None, amalgamate=False)
    assert sym.nsuper == 3
    panels, Ures = oracle.factor(A, sym, subset=[0], keep_U=True)
    np.testing.assert_array_equal(Ures[0], np.array(ex["ex4"]["U0"], dtype=float))


def test_chain_closed_form():
    n = 200
    A = G.laplacian_1d(n)
    sym = oracle.symbolic(A, None)
    L = oracle.panels_to_dense_L(sym, oracle.factor(A, sym))
    j = np.arange(n)
    np.testing.assert_allclose(np.diag(L), np.sqrt((j + 2) / (j + 1)), rtol=64 * U, atol=0)
    np.testing.assert_allclose(np.diag(L, -1), -np.sqrt((j[:-1] + 1) / (j[:-1] + 2)), rtol=64 * U, atol=0)
    assert oracle.logdet(sym, oracle.factor(A, sym)) == pytest.approx(np.log(n + 1), rel=1e-13)


@pytest.mark.parametrize("kind,dims", [("5pt", (32, 32, 1)), ("27pt", (6, 5, 4)), ("7pt", (9, 8, 7)),
                                       ("9pt", (25, 20, 1)), ("elast", (5, 5, 5))])
def test_grids_vs_dense_lapack(kind, dims):
    A, p = grid(kind, dims)
    sym = oracle.symbolic(A, p)
    panels = oracle.factor(A, sym)
    L = oracle.panels_to_dense_L(sym, panels)
    Lref, M = dense_L(A, sym)
    # M-matrix stencils are componentwise accurate; elasticity has cancellation-noise
    # entries, for which reading C11 gives the north-star bound 1e-10
    assert floored_rel(L, Lref) <= (1e-10 if kind == "elast" else 1e-12)
    # reconstruction: ||P A P^T - L L^T||_max / ||A||_max <= 100 n_f u
    nf = int(np.diff(sym.sn_rowptr).max())
    Pm = M[np.ix_(sym.perm, sym.perm)]
    assert np.abs(Pm - L @ L.T).max() / np.abs(M).max() <= 100 * nf * U
    # backward error of the solve (reading C12)
    xs = G.rhs(A.n, 0)
    b = M @ xs
    x = oracle.solve(sym, panels, b)
    be = np.abs(M @ x - b).max() / (np.abs(M).sum(axis=1).max() * np.abs(x).max() + np.abs(b).max())
    assert be <= 1e-12


@settings(max_examples=20, deadline=None)
@given(n=st.integers(1, 80), dens=st.floats(0.0, 0.25), seed=st.integers(0, 10_000))
def test_random_spd_vs_dense(n, dens, seed):
    A = G.random_spd_pattern(n, dens, seed, dup=0.3, upper=0.2)
    perm = np.random.default_rng(seed + 1).permutation(n).astype(np.int32)
    sym = oracle.symbolic(A, perm)
    L = oracle.panels_to_dense_L(sym, oracle.factor(A, sym))
    Lref, _ = dense_L(A, sym)
    assert floored_rel(L, Lref) <= 1e-12


def _eig_logdet(kind, N):
    th = np.arange(1, N + 1) * np.pi / (N + 1)
    k1 = 4 * np.sin(th / 2) ** 2          # eig of tridiag(-1,2,-1)
    t1 = 1 + 2 * np.cos(th)               # eig of tridiag(1,1,1)
    if kind == "5pt":
        lam = k1[:, None] + k1[None, :]
    elif kind == "7pt":
        lam = k1[:, None, None] + k1[None, :, None] + k1[None, None, :]
    elif kind == "9pt":
        lam = 9 - t1[:, None] * t1[None, :]
    elif kind == "27pt":
        lam = 27 - t1[:, None, None] * t1[None, :, None] * t1[None, None, :]
    return float(np.sum(np.log(lam)))


@pytest.mark.parametrize("kind,N", [("5pt", 32), ("5pt", 100), ("9pt", 60), ("7pt", 14), ("27pt", 12)])
def test_logdet_closed_form(kind, N):
    A, p = grid(kind, (N, N, N if kind in ("7pt", "27pt") else 1))
    sym = oracle.symbolic(A, p)
    ld = oracle.logdet(sym, oracle.factor(A, sym))
    assert ld == pytest.approx(_eig_logdet(kind, N), rel=1e-13)
    if (kind, N) == ("5pt", 32):
        assert ld == pytest.approx(1.210723120532049e+03, rel=1e-13)


@pytest.mark.parametrize("kind,dims", [("5pt", (20, 20, 1)), ("27pt", (7, 6, 5)), ("elast", (4, 4, 4)),
                                       ("7pt", (10, 10, 10))])
def test_manufactured_exact(kind, dims):
    """A = L0 L0^T with integer L0 (power-of-two diagonal) => L == L0 bit-exactly."""
    A0, p = grid(kind, dims)
    s0 = oracle.symbolic(A0, p, keep_struct=True)
    A, Lx = G.manufactured(A0.n, s0.Lp, s0.Li, s0.perm, seed=1234)
    sym = oracle.symbolic(A, s0.perm, keep_struct=True)
    np.testing.assert_array_equal(sym.Li, s0.Li)           # same pattern -> same symbolic
    np.testing.assert_array_equal(sym.sn_first, s0.sn_first)
    L = oracle.panels_to_dense_L(sym, oracle.factor(A, sym))
    L0 = np.zeros_like(L)
    cols = np.repeat(np.arange(A.n), np.diff(s0.Lp))
    L0[s0.Li, cols] = Lx
    np.testing.assert_array_equal(L, L0)


def test_padding_exact_zero_and_subset_consistency():
    A, p = grid("7pt", (12, 12, 12))
    sym = oracle.symbolic(A, p, keep_struct=True)
    panels = oracle.factor(A, sym)
    for s in range(sym.nsuper):
        R = sym.rows(s)
        k = sym.k(s)
        P = panels[s]
        assert (np.triu(P[:k], 1) == 0).all()
        for jj in range(k):
            j = R[jj]
            true = set(sym.Li[sym.Lp[j]:sym.Lp[j + 1]].tolist())
            pad = [ii for ii in range(jj, R.size) if R[ii] not in true]
            assert (P[pad, jj] == 0.0).all()
    # a whole subtree factored alone gives bitwise the same panels
    ch = sym.children()
    root = int(np.argmax([len(sym.rows(s)) for s in range(sym.nsuper - 1)]))
    sub, stack = [], [root]
    while stack:
        v = stack.pop(); sub.append(v); stack.extend(ch[v])
    part = oracle.factor(A, sym, subset=sub)
    for s in sub:
        np.testing.assert_array_equal(part[s], panels[s])


def test_not_spd_first_failing_column():
    A, p = grid("5pt", (16, 16, 1))
    sym = oracle.symbolic(A, p)
    for victim in (5, 77, 200):
        B = G.CSC(A.n, A.colptr, A.rowind, A.values.copy())
        d = A.colptr[victim] + np.nonzero(A.rowind[A.colptr[victim]:A.colptr[victim + 1]] == victim)[0][0]
        B.values[d] = -1.0
        M = G.full_symmetric_dense(B)[np.ix_(sym.perm, sym.perm)]
        _, info = scipy.linalg.lapack.dpotrf(M, lower=1)
        assert info > 0
        with pytest.raises(oracle.NotSPD) as e:
            oracle.factor(B, sym)
        assert e.value.col == info - 1 and e.value.orig == sym.perm[info - 1]
