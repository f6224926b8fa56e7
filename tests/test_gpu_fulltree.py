"""Full-size parity of EVERY front ("Next round" #1).

The BASELINE configs at full size, in bench.py's launch configuration
(default options, 4 concurrent branches, learned variant selector), factored
on the GPU once; then the oracle factors the WHOLE elimination tree front by
front in postorder (oracle.factor_stream: plain C, no BLAS) and every panel
is compared with the GPU's as soon as the oracle produces it -- including the
62 fronts of order > 4096 of c5 that carry 89.6% of its flops and the
14,900-pivot root.  Metric: reading C11 with the single
floor TAU of tests/_parity.py; the floored max, the unfloored max and the count
of entries below the floor are printed per config.  Plus the closed-form log
det of the Laplacian stencils and the backward error of a solve
[PAPER.md L7, L27 Sec. II-A, Fig. 1 L33-65]."""
import time

import numpy as np
import pytest

import oracle
from workloads import grids as G
from tests._parity import ParityStats, TOL_L
from tests.test_gpu_parity import backward_error, spmv

pytestmark = pytest.mark.gpu

TOL_BE = 1e-12


def _closed_form_logdet(kind, N):
    th = np.arange(1, N + 1) * np.pi / (N + 1)
    t1 = 1 + 2 * np.cos(th)
    k1 = 4 * np.sin(th / 2) ** 2
    lam = {"27pt": lambda: 27 - t1[:, None, None] * t1[None, :, None] * t1[None, None, :],
           "9pt": lambda: 9 - t1[:, None] * t1[None, :],
           "7pt": lambda: k1[:, None, None] + k1[None, :, None] + k1[None, None, :]}.get(kind)
    return None if lam is None else float(np.sum(np.log(lam())))


@pytest.mark.parametrize("name", ["c5", "c4", "c3", "c2"])
def test_full_tree_parity(name):
    import torch
    assert torch.cuda.is_available()
    import paper_conf_ipps_georgesgsc11_b200 as mf
    c = G.CONFIGS[name]
    A, p = G.make_config(c["kind"], c["N"])
    S = mf.Solver()
    S.analyze(A.n, A.colptr, A.rowind, p)
    S.factor(A.values)
    sym = oracle.symbolic(A, p)
    m_matrix = c["kind"] != "elast"
    st = ParityStats()
    big = 0
    t0 = time.perf_counter()
    for s, Po in oracle.factor_stream(A, sym):
        f, k = Po.shape
        st.add(s, S.panel(s, f, k), Po, m_matrix=m_matrix)
        big += f > 4096
    rep = st.report()
    print(f"{name}: {rep} fronts>4096={big} oracle+compare {time.perf_counter() - t0:.1f}s")
    assert st.panels == sym.nsuper
    assert rep["floored_max"] <= TOL_L, rep
    if m_matrix:   # no cancellation: componentwise accurate, padding exactly 0 (reading C10)
        assert rep["unfloored_max"] <= TOL_L, rep
        assert st.pad_violations == 0, rep
    ld = _closed_form_logdet(c["kind"], c["N"])
    if ld is not None:
        assert 2 * np.sum(np.log(S.diag())) == pytest.approx(ld, rel=1e-12)
    b = spmv(A, G.rhs(A.n, 0))
    x = S.solve(b)
    assert backward_error(A, x, b) <= TOL_BE
