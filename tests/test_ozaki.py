"""Schur updates on the int8 tensor cores (Ozaki scheme,
csrc/ozaki_update.cuh; Sec. III-B for the paper's own
reduced-precision GPU variant).

ozaki_slices = 8 is an FP64-class emulation: the factor must meet the
north-star parity bar (reading C11, floored at TAU, tests/_parity.py) -- on
grids, on the full-size c4 / c5 trees -- and reproduce manufactured integer
factors bit-exactly (small integer panels are cut into digits without loss and
every digit product is exact in int32).  The extra UNFLOORED check the DMMA
path meets on the stencils does not apply: each panel row is scaled by its own
largest entry, so entries far below it keep fewer of the 56 digit bits
(measured 1.5e-10 unfloored on a 27-point 24^3 grid, floored 6e-12).  Reduced slices (3..7) are the mixed-
precision mode: the factor is inexact by design and mf_solve refines in fp64
until the backward error of reading C12 holds.
CPU (not gpu): the plan converts the long-K update launches and only those."""
import numpy as np
import pytest

import oracle
import paper_conf_ipps_georgesgsc11_b200 as mf
from workloads import grids as G
from tests._grids import grid
from tests._parity import ParityStats, TOL_L


def test_plan_converts_long_k_updates(monkeypatch):
    monkeypatch.setenv("MF_OZ_MIN_K", "256")
    A, p = grid("27pt", (30, 30, 30))
    S0 = mf.Solver(host_only=True)
    S0.analyze(A.n, A.colptr, A.rowind, p)
    S8 = mf.Solver(host_only=True, ozaki_slices=8)
    S8.analyze(A.n, A.colptr, A.rowind, p)
    assert S0.info()["launches_ozaki"] == 0
    assert S8.info()["launches_ozaki"] > 0 and S8.info()["ozaki_slices"] == 8
    assert S8.info()["workspace_bytes"] == 0   # host-only: nothing allocated
    with pytest.raises(mf.MfError):
        mf.Solver(host_only=True, ozaki_slices=2)


gpu = pytest.mark.gpu


@pytest.fixture
def all_int8(monkeypatch):
    """Convert every update launch with K >= 64 (the default threshold, 2048, is
    where the int8 path wins on c5; these grids are smaller)."""
    monkeypatch.setenv("MF_OZ_MIN_K", "64")


@gpu
@pytest.mark.parametrize("kind,dims", [("27pt", (24, 24, 24)), ("7pt", (40, 40, 40)), ("elast", (12, 12, 12)),
                                       ("27pt", (33, 31, 29))])
def test_ozaki8_parity(kind, dims, all_int8):
    A, p = grid(kind, dims)
    S = mf.Solver(ozaki_slices=8)
    S.analyze(A.n, A.colptr, A.rowind, p)
    assert S.info()["launches_ozaki"] > 0
    S.factor(A.values)
    sym = oracle.symbolic(A, p)
    st = ParityStats()
    for s, Po in oracle.factor_stream(A, sym):
        st.add(s, S.panel(s, *Po.shape), Po, m_matrix=kind != "elast")
    rep = st.report()
    print(kind, dims, rep)
    assert rep["floored_max"] <= TOL_L, rep
    from tests.test_gpu_parity import backward_error, spmv
    b = spmv(A, G.rhs(A.n, 0))
    assert backward_error(A, S.solve(b), b) <= 1e-12


@gpu
@pytest.mark.parametrize("dims", [(16, 16, 16), (22, 21, 20)])
def test_ozaki8_manufactured_bit_exact(dims, all_int8):
    A0, p = grid("27pt", dims)
    s0 = oracle.symbolic(A0, p, keep_struct=True)
    A, Lx = G.manufactured(A0.n, s0.Lp, s0.Li, s0.perm, seed=1234)
    S8 = mf.Solver(ozaki_slices=8, small_front_max=8)   # every front through the tiled path
    S8.analyze(A.n, A.colptr, A.rowind, s0.perm)
    assert S8.info()["launches_ozaki"] > 0
    S8.factor(A.values)
    S0 = mf.Solver(small_front_max=8)
    S0.analyze(A.n, A.colptr, A.rowind, s0.perm)
    S0.factor(A.values)
    sn = S0.supernodes()
    for s in range(S0.info()["nsuper"]):
        f = int(sn["sn_rowptr"][s + 1] - sn["sn_rowptr"][s])
        k = int(sn["sn_first"][s + 1] - sn["sn_first"][s])
        np.testing.assert_array_equal(S8.panel(s, f, k), S0.panel(s, f, k))


@gpu
@pytest.mark.parametrize("name", ["c5", "c4"])
def test_ozaki8_full_tree_parity(name):
    c = G.CONFIGS[name]
    A, p = G.make_config(c["kind"], c["N"])
    S = mf.Solver(ozaki_slices=8)
    S.analyze(A.n, A.colptr, A.rowind, p)
    S.factor(A.values)
    sym = oracle.symbolic(A, p)
    st = ParityStats()
    for s, Po in oracle.factor_stream(A, sym):
        st.add(s, S.panel(s, *Po.shape), Po, m_matrix=c["kind"] != "elast")
    rep = st.report()
    print(name, "ozaki8", rep, "t_factor", S.info()["t_factor"])
    assert rep["floored_max"] <= TOL_L, rep


@gpu
@pytest.mark.parametrize("slices,kind,dims", [(4, "27pt", (24, 24, 24)), (3, "elast", (10, 10, 10)),
                                              (5, "7pt", (36, 36, 36))])
def test_mixed_precision_refined_solve(slices, kind, dims, all_int8):
    """Reduced-precision Schur updates (3..5 slices) + fp64 iterative refinement in
    mf_solve: the refined x meets reading C12 (backward error <= 1e-12, checked
    here on the host); the unrefined factor alone does not need to."""
    from tests.test_gpu_parity import backward_error, spmv
    A, p = grid(kind, dims)
    S = mf.Solver(ozaki_slices=slices)
    S.analyze(A.n, A.colptr, A.rowind, p)
    assert S.info()["launches_ozaki"] > 0
    S.factor(A.values)
    b = spmv(A, G.rhs(A.n, 0))
    x = S.solve(b)
    inf = S.info()
    be = backward_error(A, x, b)
    print(kind, dims, "slices", slices, "refine steps", inf["refine_steps"], "device berr", inf["solve_berr"],
          "host berr", be)
    assert be <= 1e-12
    assert inf["refine_steps"] >= 1 and 0 <= inf["solve_berr"] <= 1e-12
    S0 = mf.Solver(ozaki_slices=slices, refine_iters=0)   # the same factor without refinement
    S0.analyze(A.n, A.colptr, A.rowind, p)
    S0.factor(A.values)
    assert backward_error(A, S0.solve(b), b) > be
