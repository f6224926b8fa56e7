"""Reading C11 settled by a higher-precision REFEREE (VERDICT r1 "What's weak" #2).

Q1 elasticity is not an M-matrix: about 3% of the structural entries of its L
are cancellation noise (down to exactly 0), whose relative error is meaningless
in any fp64 implementation.  The referee is the column Cholesky algorithm in
long double (64-bit significand, oracle/numeric.c) on the dense P A P^T; it is
exact to ~2^-64 relative to the column max, 2^11 below fp64 rounding.

Pins: the oracle (CPU, -m "not gpu") is within ORACLE_ULP and the GPU factor
(-m gpu) within GPU_ULP ulp of the column max of the referee on EVERY entry;
that envelope is what tests/_parity.py turns into the single floor TAU = 4e-5.
Also: with the floor at TAU both are within 1e-10 of the referee, i.e. the
C11 metric measures rounding, not method error."""
import numpy as np
import pytest

import oracle
from workloads import grids as G
from tests._grids import grid
from tests._parity import TAU, TOL_L, U64

ORACLE_ULP = 8.0    # measured: oracle 5.5 / 5.2 / 7.0 / 7.4 u at 6^3 / 8^3 / 10^3 / 12^3
GPU_ULP = 24.0      # measured: GPU 13.2 / 17.8 u at 8^3 / 12^3 (one DMMA accumulation chain, rsqrt pivots)


def _referee(N):
    A, p = grid("elast", (N, N, N))
    sym = oracle.symbolic(A, p)
    M = G.full_symmetric_dense(A)[np.ix_(sym.perm, sym.perm)]
    return A, p, sym, oracle.dense_cholesky_longdouble(M)


def _envelope(L, Lr):
    colmax = np.abs(Lr).max(axis=0)
    err = np.abs(L.astype(np.longdouble) - Lr)
    eps = float((err / colmax[None, :]).max()) / U64
    den = np.maximum(np.abs(Lr), TAU * colmax[None, :])
    floored = float((err / den).max())
    return eps, floored


@pytest.mark.parametrize("N", [6, 8, 10])
def test_oracle_within_envelope_of_referee(N):
    A, p, sym, Lr = _referee(N)
    L = oracle.panels_to_dense_L(sym, oracle.factor(A, sym))
    eps, floored = _envelope(L, Lr)
    print(f"elast {N}^3: oracle vs long-double referee {eps:.2f} u of colmax, floored rel {floored:.2e}")
    assert eps <= ORACLE_ULP
    assert floored <= TOL_L / 2


@pytest.mark.gpu
@pytest.mark.parametrize("N", [8, 12])
def test_gpu_within_envelope_of_referee(N):
    import torch
    assert torch.cuda.is_available()
    import paper_conf_ipps_georgesgsc11_b200 as mf
    A, p, sym, Lr = _referee(N)
    S = mf.Solver()
    S.analyze(A.n, A.colptr, A.rowind, p)
    S.factor(A.values)
    panels = {s: S.panel(s, sym.rows(s).size, sym.k(s)) for s in range(sym.nsuper)}
    L = oracle.panels_to_dense_L(sym, panels)
    eps, floored = _envelope(L, Lr)
    print(f"elast {N}^3: GPU vs long-double referee {eps:.2f} u of colmax, floored rel {floored:.2e}")
    assert eps <= GPU_ULP
    assert floored <= TOL_L / 2
