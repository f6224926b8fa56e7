"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle,
element by element, on seeded synthetic inputs.

Tolerances (north star, BASELINE.json): max relative entry error of L vs the
oracle <= 1e-10 under reading C11 (one floor, tests/_parity.py TAU);
amalgamation padding exactly 0.0 (reading C10); backward error
||Ax - b||_inf / (||A||_inf ||x||_inf + ||b||_inf) <= 1e-12 (reading C12);
manufactured integer factors bit-exact.
"""
import numpy as np
import pytest

import oracle
from workloads import grids as G
from tests._grids import dense_from_rows, grid
from tests._parity import TAU

pytestmark = pytest.mark.gpu

TOL_L = 1e-10
TOL_BE = 1e-12


@pytest.fixture(scope="module")
def mf():
    import torch
    assert torch.cuda.is_available(), "GPU tests need a CUDA device"
    import paper_conf_ipps_georgesgsc11_b200 as m
    return m


def c11(Pg, Po, tau=TAU):
    """Reading C11 floored relative error of one panel (columns = columns of L)."""
    colmax = np.abs(Po).max(axis=0)
    den = np.maximum(np.abs(Po), tau * colmax[None, :])
    den[den == 0] = 1.0
    return float((np.abs(Pg - Po) / den).max())


def factor_both(mf, A, perm, supernodes=None, **opts):
    S = mf.Solver(**opts)
    S.analyze(A.n, A.colptr, A.rowind, perm)
    S.factor(A.values)
    sym = oracle.symbolic(A, perm, keep_struct=A.n <= 200_000)
    panels = oracle.factor(A, sym, subset=supernodes)
    return S, sym, panels


def check_panels(S, sym, panels, exact=False, tau=TAU):
    worst = 0.0
    for s, Po in panels.items():
        f, k = Po.shape
        Pg = S.panel(s, f, k)
        assert (np.triu(Pg[:k], 1) == 0).all()
        if exact:
            np.testing.assert_array_equal(Pg, Po)
        else:
            worst = max(worst, c11(Pg, Po, tau))
        if sym.Li is not None:   # amalgamation padding must be exactly 0
            R = sym.rows(s)
            for jj in range(k):
                j = R[jj]
                st = sym.Li[sym.Lp[j]:sym.Lp[j + 1]]
                pad = np.setdiff1d(np.arange(jj, f), np.searchsorted(R, st))
                assert (Pg[pad, jj] == 0.0).all()
    assert worst <= TOL_L, worst
    return worst


def backward_error(A, x, b):
    M_lower = (A.colptr, A.rowind, A.values)
    n = A.n
    cols = np.repeat(np.arange(n), np.diff(A.colptr))
    r = A.rowind.astype(np.int64)
    keep = r >= cols
    r, c, v = r[keep], cols[keep], A.values[keep]
    Ax = np.zeros(n)
    np.add.at(Ax, r, v * x[c])
    off = r != c
    np.add.at(Ax, c[off], v[off] * x[r[off]])
    rowabs = np.zeros(n)
    np.add.at(rowabs, r, np.abs(v))
    np.add.at(rowabs, c[off], np.abs(v[off]))
    del M_lower
    return np.abs(Ax - b).max() / (rowabs.max() * np.abs(x).max() + np.abs(b).max())


def spmv(A, x):
    n = A.n
    cols = np.repeat(np.arange(n), np.diff(A.colptr))
    r = A.rowind.astype(np.int64)
    keep = r >= cols
    r, c, v = r[keep], cols[keep], A.values[keep]
    y = np.zeros(n)
    np.add.at(y, r, v * x[c])
    off = r != c
    np.add.at(y, c[off], v[off] * x[r[off]])
    return y


CASES = [("5pt", (32, 32, 1)), ("27pt", (6, 5, 4)), ("7pt", (12, 12, 12)), ("9pt", (60, 45, 1)),
         ("elast", (6, 6, 6)), ("27pt", (16, 16, 16)), ("7pt", (24, 24, 24)), ("27pt", (21, 19, 17))]


@pytest.mark.parametrize("kind,dims", CASES)
def test_grid_parity(mf, kind, dims):
    A, p = grid(kind, dims)
    S, sym, panels = factor_both(mf, A, p)
    worst = check_panels(S, sym, panels)
    b = spmv(A, G.rhs(A.n, 0))
    x = S.solve(b)
    assert backward_error(A, x, b) <= TOL_BE
    ld_g = 2 * np.sum(np.log(S.diag()))
    assert ld_g == pytest.approx(oracle.logdet(sym, panels), rel=1e-12)
    print(kind, dims, "max C11 rel err", worst)


@pytest.mark.parametrize("small_max,w", [(8, 64), (8, 16), (48, 32), (160, 64)])
def test_variant_paths_agree(mf, small_max, w):
    """Force fronts through the tiled path (small_max=8) or the fused SMEM kernel
    (160): both must match the oracle."""
    A, p = grid("27pt", (14, 13, 12))
    S, sym, panels = factor_both(mf, A, p, small_front_max=small_max, panel_w=w)
    check_panels(S, sym, panels)
    b = spmv(A, G.rhs(A.n, 0))   # the solve's dataflow tasks with w-column blocks (w | 64)
    assert backward_error(A, S.solve(b), b) <= TOL_BE


@pytest.mark.parametrize("n", [1, 2, 63, 64, 65, 200, 1000, 2500])
def test_dense_and_chain(mf, n):
    """One supernode (dense: k = n, m = 0 -> blocked potrf with ragged last block)
    and the 1D chain (relaxed into one front)."""
    rng = np.random.default_rng(n)
    X = rng.standard_normal((n, n))
    D = X @ X.T / n + np.eye(n)
    A = dense_from_rows(D)
    S, sym, panels = factor_both(mf, A, np.arange(n, dtype=np.int32))
    check_panels(S, sym, panels)
    C = G.laplacian_1d(n)
    S2, sym2, panels2 = factor_both(mf, C, np.arange(n, dtype=np.int32))
    check_panels(S2, sym2, panels2)


@pytest.mark.parametrize("kind,dims,small_max", [("5pt", (30, 30, 1), 128), ("27pt", (12, 12, 12), 128),
                                                 ("elast", (5, 5, 5), 128), ("7pt", (16, 16, 16), 128),
                                                 ("27pt", (12, 12, 12), 8), ("27pt", (10, 9, 11), 160)])
def test_manufactured_bit_exact(mf, kind, dims, small_max):
    A0, p = grid(kind, dims)
    s0 = oracle.symbolic(A0, p, keep_struct=True)
    A, Lx = G.manufactured(A0.n, s0.Lp, s0.Li, s0.perm, seed=1234)
    S = mf.Solver(small_front_max=small_max)
    S.analyze(A.n, A.colptr, A.rowind, s0.perm)
    S.factor(A.values)
    sym = oracle.symbolic(A, s0.perm, keep_struct=True)
    # expected panels straight from L0 (no oracle arithmetic involved)
    for s in range(sym.nsuper):
        R = sym.rows(s)
        k = sym.k(s)
        exp = np.zeros((R.size, k))
        for jj in range(k):
            j = R[jj]
            st = s0.Li[s0.Lp[j]:s0.Lp[j + 1]]
            exp[np.searchsorted(R, st), jj] = Lx[s0.Lp[j]:s0.Lp[j + 1]]
        np.testing.assert_array_equal(S.panel(s, R.size, k), exp)


@pytest.mark.parametrize("seed", [0, 1, 2, 3])
def test_random_spd_with_duplicates(mf, seed):
    n = [50, 300, 900, 1500][seed]
    A = G.random_spd_pattern(n, 0.02 if n > 500 else 0.08, seed, dup=0.3, upper=0.2)
    perm = np.random.default_rng(seed).permutation(n).astype(np.int32)
    S, sym, panels = factor_both(mf, A, perm)
    check_panels(S, sym, panels)


def test_not_spd_reports_first_failing_column(mf):
    A, p = grid("27pt", (12, 12, 12))
    sym = oracle.symbolic(A, p)
    S = mf.Solver()
    S.analyze(A.n, A.colptr, A.rowind, p)
    for victim in (7, 900, int(sym.perm[-1])):
        B = G.CSC(A.n, A.colptr, A.rowind, A.values.copy())
        d = A.colptr[victim] + np.nonzero(A.rowind[A.colptr[victim]:A.colptr[victim + 1]] == victim)[0][0]
        B.values[d] = -50.0
        with pytest.raises(oracle.NotSPD) as e:
            oracle.factor(B, sym)
        with pytest.raises(mf.MfNotSPD) as g:
            S.factor(B.values)
        assert g.value.failed_col == e.value.orig
        with pytest.raises(mf.MfError):
            S.solve(np.ones(A.n))
    S.factor(A.values)             # recovers with valid values
    S.solve(np.ones(A.n))


def test_device_pointers_and_refactor(mf):
    import torch
    A, p = grid("27pt", (15, 15, 15))
    S = mf.Solver()
    S.analyze(A.n, A.colptr, A.rowind, p)
    S.factor(A.values)
    b = spmv(A, G.rhs(A.n, 0))
    x_host = S.solve(b)
    vals_d = torch.from_numpy(A.values).cuda()
    S.factor(vals_d)
    b_d = torch.from_numpy(b).cuda()
    x_d = torch.empty_like(b_d)
    S.solve(b_d, x_d)
    np.testing.assert_array_equal(x_d.cpu().numpy(), x_host)   # deterministic
    # refactor with scaled values: L scales by sqrt(4) = 2 exactly
    S.factor(A.values * 4.0)
    np.testing.assert_array_equal(S.solve(b), x_host / 4.0)


def test_deterministic_bitwise(mf):
    A, p = grid("27pt", (18, 18, 18))
    S = mf.Solver()
    S.analyze(A.n, A.colptr, A.rowind, p)
    inf = S.info()
    outs = []
    for _ in range(3):
        S.factor(A.values)
        outs.append(S.export_panels(sum_panel_words(S, inf)))
    assert all(np.array_equal(outs[0], o) for o in outs[1:])


@pytest.mark.parametrize("kind,dims,small_max,w", [("27pt", (18, 18, 18), 128, 64), ("7pt", (24, 24, 24), 8, 64),
                                                    ("elast", (9, 9, 9), 48, 32), ("9pt", (90, 70, 1), 8, 16)])
def test_fused_extend_add_bit_identical(mf, kind, dims, small_max, w):
    """the extend-add of the U^s part fused into the syrk prologue
    sums 0 + U^c1 + U^c2 ... per element in the assembly kernel's order (reading
    C6), so L is bit-identical with fuse_ea on and off (odd and even k, shifted
    problems, small and tiled children) -- and both match the oracle."""
    A, p = grid(kind, dims)
    outs = []
    for fuse in (False, True):
        S = mf.Solver(fuse_ea=fuse, small_front_max=small_max, panel_w=w)
        S.analyze(A.n, A.colptr, A.rowind, p)
        inf = S.info()
        S.factor(A.values)
        outs.append(S.export_panels(sum_panel_words(S, inf)))
    np.testing.assert_array_equal(outs[0], outs[1])
    sym = oracle.symbolic(A, p, keep_struct=True)
    check_panels(S, sym, oracle.factor(A, sym))


@pytest.mark.parametrize("kind,dims,nb", [("27pt", (24, 24, 24), 1), ("7pt", (32, 32, 32), 4), ("elast", (10, 10, 10), 1)])
def test_lookahead_bit_identical(mf, kind, dims, nb):
    """Look-ahead (trailing updates split so the next panel runs beside the rest on
    a side stream) changes only the schedule: L is bitwise equal with it on and
    off, and matches the oracle."""
    A, p = grid(kind, dims)
    outs = []
    for la in (False, True, True):
        S = mf.Solver(lookahead=la, nbranch=nb)
        S.analyze(A.n, A.colptr, A.rowind, p)
        inf = S.info()
        S.factor(A.values)
        outs.append(S.export_panels(sum_panel_words(S, inf)))
    np.testing.assert_array_equal(outs[0], outs[1])
    np.testing.assert_array_equal(outs[0], outs[2])
    sym = oracle.symbolic(A, p, keep_struct=True)
    check_panels(S, sym, oracle.factor(A, sym))


_BULK_CHILD = r'''
import hashlib, sys
sys.path.insert(0, ".")
import numpy as np
import paper_conf_ipps_georgesgsc11_b200 as mf
from tests._grids import grid
kind, dims, sm = sys.argv[1], tuple(int(x) for x in sys.argv[2].split(",")), int(sys.argv[3])
A, p = grid(kind, dims)
S = mf.Solver(small_front_max=sm, nbranch=1)
S.analyze(A.n, A.colptr, A.rowind, p)
S.factor(A.values)
sn = S.supernodes()
k = np.diff(sn["sn_first"]); f = np.diff(sn["sn_rowptr"])
h = hashlib.sha256(S.export_panels(int(np.sum(f * k))).tobytes())
h.update(S.solve(np.ones(A.n)).tobytes())
print(h.hexdigest())
'''


@pytest.mark.parametrize("kind,dims,sm", [("27pt", (20, 20, 20), 8), ("7pt", (28, 28, 28), 128),
                                         ("elast", (9, 9, 9), 48)])
def test_nan_filled_arenas_bit_identical(mf, kind, dims, sm):
    """Debug NaN-fill (MF_DEBUG_NANFILL=1): with the L / U / vector arenas filled with
    NaN at analyze instead of zeros, L is bitwise the same -- no kernel reads a word
    into a real output before this factorization wrote it (VERDICT r1 hygiene)."""
    import os
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    out = []
    for e in ({}, dict(MF_DEBUG_NANFILL="1")):
        r = subprocess.run([sys.executable, "-c", _BULK_CHILD, kind, ",".join(map(str, dims)), str(sm)], cwd=root,
                           env=dict(os.environ, **e), capture_output=True, text=True, timeout=600)
        assert r.returncode == 0, r.stderr[-2000:]
        out.append(r.stdout.strip().splitlines()[-1])
    assert out[0] == out[1], out


@pytest.mark.parametrize("kind,dims,sm", [("27pt", (20, 20, 20), 8), ("7pt", (28, 28, 28), 128)])
def test_bulk_staging_bit_identical(mf, kind, dims, sm):
    """The DMMA update's operand-staging variants (per-thread cp.async with CTA
    barriers, 3 or 2 stages; warp-0 bulk copies with full/empty mbarriers)
    compute every element in the same order, so L is bitwise equal with any of
    them forced on every launch (MF_UPD_BULK / MF_UPD_LOWK = 0/1; the default
    picks per launch).  Guards the
    generic-read -> async-write hazard on the ring slots."""
    import os
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    out = []
    envs = [dict(MF_UPD_BULK="0", MF_UPD_LOWK="0"), dict(MF_UPD_BULK="1"), dict(MF_UPD_BULK="1"),
            dict(MF_UPD_BULK="0", MF_UPD_LOWK="1"), {}, dict(MF_U_REUSE="0")]   # + U slots not recycled
    for e in envs:
        r = subprocess.run([sys.executable, "-c", _BULK_CHILD, kind, ",".join(map(str, dims)), str(sm)], cwd=root,
                           env=dict(os.environ, **e), capture_output=True, text=True, timeout=600)
        assert r.returncode == 0, r.stderr[-2000:]
        out.append(r.stdout.strip().splitlines()[-1])
    assert len(set(out)) == 1, out


def sum_panel_words(S, inf):
    sn = S.supernodes()
    k = np.diff(sn["sn_first"]).astype(np.int64)
    f = np.diff(sn["sn_rowptr"]).astype(np.int64)
    return int((k * f).sum())


@pytest.mark.parametrize("nb", [1, 4])
def test_profiling_modes_same_factor(mf, nb):
    """Eager per-launch timing (profiling 1) and the concurrent-graph timeline
    (profiling 2: timing events captured into the graph) only observe: L is bitwise
    equal to the plain graph's; every launch of the timeline ends after it starts,
    the launches of one stream run in program order, and the per-launch times of
    both modes are positive."""
    A, p = grid("7pt", (24, 24, 24))
    outs = []
    for mode in (0, 1, 2):
        S = mf.Solver(nbranch=nb)
        S.analyze(A.n, A.colptr, A.rowind, p)
        inf = S.info()
        S.set_profiling(mode)
        S.factor(A.values)
        S.factor(A.values)
        outs.append(S.export_panels(sum_panel_words(S, inf)))
        if mode == 1:
            assert (S.launch_times() > 0).all()
        if mode == 2:
            t0, t1 = S.launch_timeline()
            prog = S.program()
            assert len(t0) == len(prog) and (t1 >= t0).all() and (t0 >= 0).all()
            for st in {L["stream"] for L in prog}:
                idx = [i for i, L in enumerate(prog) if L["stream"] == st]
                assert (np.diff(t1[idx]) >= 0).all()
            assert all(k["launches"] > 0 for k in S.kernel_stats() if k["ms"] > 0)
        else:
            with pytest.raises(mf.MfError):
                S.launch_timeline()
    np.testing.assert_array_equal(outs[0], outs[1])
    np.testing.assert_array_equal(outs[0], outs[2])


def test_degenerate_inputs(mf):
    # n = 1
    A = dense_from_rows([[9.0]])
    S = mf.Solver()
    S.analyze(1, A.colptr, A.rowind, np.zeros(1, dtype=np.int32))
    S.factor(A.values)
    assert S.diag()[0] == 3.0
    np.testing.assert_array_equal(S.solve(np.array([18.0])), [2.0])
    # missing diagonal => not SPD at that (original) column
    A, p = grid("5pt", (6, 6, 1))
    keep = ~((A.rowind == 10) & (np.repeat(np.arange(A.n), np.diff(A.colptr)) == 10))
    cols = np.repeat(np.arange(A.n), np.diff(A.colptr))[keep]
    colptr = np.zeros(A.n + 1, dtype=np.int64)
    np.cumsum(np.bincount(cols, minlength=A.n), out=colptr[1:])
    B = G.CSC(A.n, colptr, A.rowind[keep], A.values[keep])
    S = mf.Solver()
    S.analyze(B.n, B.colptr, B.rowind, p)
    with pytest.raises(mf.MfNotSPD):
        S.factor(B.values)
    # empty matrix
    S = mf.Solver()
    S.analyze(0, np.zeros(1, dtype=np.int64), np.zeros(0, dtype=np.int32), np.zeros(0, dtype=np.int32))
    S.factor(np.zeros(0))
    assert S.solve(np.zeros(0)).size == 0




@pytest.mark.parametrize("kind,dims", [("27pt", (16, 15, 14)), ("elast", (7, 7, 7))])
def test_null_perm_parity(mf, kind, dims):
    """perm == NULL (library METIS ordering): the factor under the returned final
    perm matches the oracle's, and the solve is backward stable."""
    A, _ = grid(kind, dims)
    S = mf.Solver()
    S.analyze(A.n, A.colptr, A.rowind, None)
    S.factor(A.values)
    fp = S.perm()
    sym = oracle.symbolic(A, fp, keep_struct=True)
    check_panels(S, sym, oracle.factor(A, sym))
    b = spmv(A, G.rhs(A.n, 0))
    assert backward_error(A, S.solve(b), b) <= TOL_BE


def test_export_csc_matches_panels_and_oracle(mf):
    """mf_export_L: supernodal CSC of L; every column equals the oracle's
    (reading C11), padding rows exactly 0, L L^T reconstructs P A P^T."""
    A, p = grid("27pt", (11, 10, 9))
    S = mf.Solver()
    S.analyze(A.n, A.colptr, A.rowind, p)
    S.factor(A.values)
    Lp, Li, Lx = S.export_L()
    sym = oracle.symbolic(A, p, keep_struct=True)
    panels = oracle.factor(A, sym)
    Lo = oracle.panels_to_dense_L(sym, panels)
    Lg = np.zeros_like(Lo)
    cols = np.repeat(np.arange(A.n), np.diff(Lp))
    Lg[Li, cols] = Lx
    assert c11(Lg, Lo) <= TOL_L
    M = G.full_symmetric_dense(A)[np.ix_(sym.perm, sym.perm)]
    assert np.abs(Lg @ Lg.T - M).max() <= 1e-12 * np.abs(M).max()


def test_torch_allocator_hooks(mf):
    """mf_options.dev_alloc / dev_free routed to PyTorch's caching allocator: the
    arena comes from torch (its reserved memory grows) and L is bitwise the same."""
    import torch
    A, p = grid("27pt", (16, 16, 16))
    outs = []
    for ta in (False, True):
        torch.cuda.synchronize()
        before = torch.cuda.memory_allocated()
        S = mf.Solver(torch_alloc=ta)
        S.analyze(A.n, A.colptr, A.rowind, p)
        grew = torch.cuda.memory_allocated() - before
        assert (grew >= S.info()["workspace_bytes"] // 2) if ta else grew == 0
        S.factor(A.values)
        outs.append(S.export_panels(sum_panel_words(S, S.info())))
        S.close()
        if ta:
            assert torch.cuda.memory_allocated() == before   # every block returned
    np.testing.assert_array_equal(outs[0], outs[1])


def test_solve_nrhs(mf):
    """mf_solve_nrhs: X(:, r) = A^{-1} B(:, r), bitwise equal to one mf_solve per
    column; host and device buffers."""
    import torch
    A, p = grid("27pt", (15, 14, 13))
    S = mf.Solver()
    S.analyze(A.n, A.colptr, A.rowind, p)
    S.factor(A.values)
    rng = np.random.default_rng(5)
    B = np.asfortranarray(rng.uniform(-1, 1, (A.n, 5)))
    X = S.solve_nrhs(B)
    for r in range(5):
        np.testing.assert_array_equal(X[:, r], S.solve(np.ascontiguousarray(B[:, r])))
        assert backward_error(A, X[:, r], B[:, r]) <= TOL_BE
    Bt = torch.from_numpy(np.ascontiguousarray(B.T)).cuda()   # (nrhs, n) rows = columns of B
    Xt = S.solve_nrhs(Bt)
    np.testing.assert_array_equal(Xt.cpu().numpy().T, X)


def test_solve_tall_tails(mf):
    """Dataflow solve with fronts whose update part spans more than 16 slabs of 64
    rows (the backward tail-segment tasks, kernels.cu bsolve_cols_task) and with a
    several-chunk init: backward stable, and nrhs bitwise equal to single solves."""
    A, p = grid("7pt", (40, 40, 40))
    S = mf.Solver()
    S.analyze(A.n, A.colptr, A.rowind, p)
    S.factor(A.values)
    sn = S.supernodes()
    k = np.diff(sn["sn_first"])
    f = np.diff(sn["sn_rowptr"])
    assert (f - k > 16 * 64).any() and (f > 2048).any()
    B = np.asfortranarray(np.stack([spmv(A, G.rhs(A.n, r)) for r in range(3)], axis=1))
    X = S.solve_nrhs(B)
    for r in range(3):
        x = S.solve(np.ascontiguousarray(B[:, r]))
        assert backward_error(A, x, B[:, r]) <= TOL_BE
        np.testing.assert_array_equal(X[:, r], x)
