"""CPU-side checks of the product boundary (no compute calls without a GPU):
libmf.so loads and exports every symbol include/mf.h declares, and the host
symbolic layer (run in host-only mode) matches the oracle BIT-EXACTLY
(north star: "The symbolic outputs (etree, supernode partition, nnz(L)) must
match bit-exact")."""
import ctypes
import os
import re

import numpy as np
import pytest
from hypothesis import given, settings, strategies as st

import oracle
import paper_conf_ipps_georgesgsc11_b200 as mf
from workloads import grids as G
from tests._grids import grid

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def declared_symbols():
    hdr = open(os.path.join(ROOT, "include", "mf.h")).read()
    return sorted(set(re.findall(r"\b(mf_[A-Za-z_]+)\s*\(", hdr)))


def test_library_exports_every_declared_symbol():
    lib = ctypes.CDLL(mf.lib_path())
    decl = declared_symbols()
    assert set(decl) == set(mf.EXPORTED_SYMBOLS)
    for name in decl:
        assert hasattr(lib, name), name


def test_strerror_and_defaults():
    assert mf.lib.mf_strerror(mf.MF_NOT_SPD) == b"matrix is not symmetric positive definite"
    o = mf.Options()
    assert mf.lib.mf_default_options(ctypes.byref(o)) == 0
    assert list(o.nrelax) == [4, 16, 48] and list(o.zrelax) == [0.8, 0.1, 0.05]
    assert o.fuse_ea == 1 and o.nbranch == 4 and o.lookahead == 0
    assert mf.lib.mf_default_options(None) == mf.MF_ERR_ARG


def _check_symbolic(A, perm, **kw):
    S = mf.Solver(host_only=True, amalgamate=kw.get("amalgamate", True))
    S.analyze(A.n, A.colptr, A.rowind, perm)
    so = oracle.symbolic(A, perm, amalgamate=kw.get("amalgamate", True))
    par, cc = S.etree()
    sn = S.supernodes()
    inf = S.info()
    np.testing.assert_array_equal(S.perm(), so.perm)
    np.testing.assert_array_equal(par, so.parent)
    np.testing.assert_array_equal(cc, so.cc)
    np.testing.assert_array_equal(sn["fund_first"], so.fund_first)
    np.testing.assert_array_equal(sn["sn_first"], so.sn_first)
    np.testing.assert_array_equal(sn["sn_parent"], so.sn_parent)
    np.testing.assert_array_equal(sn["sn_rowptr"], so.sn_rowptr)
    np.testing.assert_array_equal(sn["sn_rows"], so.sn_rows)
    assert inf["nnzL"] == so.nnzL and inf["flops_true"] == so.flops
    assert inf["nnzL_stored"] == so.stored_L and inf["flops_exec"] == so.exec_flops
    assert inf["nsuper"] == so.nsuper and inf["nfund"] == so.nfund
    S.close()
    return inf


@pytest.mark.parametrize("kind,dims", [("5pt", (32, 32, 1)), ("27pt", (6, 5, 4)), ("7pt", (12, 12, 12)),
                                       ("9pt", (40, 33, 1)), ("elast", (6, 6, 6)), ("27pt", (20, 20, 20)),
                                       ("7pt", (64, 64, 64))])
def test_symbolic_bit_exact_vs_oracle(kind, dims):
    A, p = grid(kind, dims)
    _check_symbolic(A, p)
    _check_symbolic(A, p, amalgamate=False)


@settings(max_examples=30, deadline=None)
@given(n=st.integers(1, 300), dens=st.floats(0.0, 0.1), seed=st.integers(0, 10_000), shuffle=st.booleans())
def test_symbolic_random_patterns(n, dens, seed, shuffle):
    A = G.random_spd_pattern(n, dens, seed, dup=0.2, upper=0.1)
    perm = np.random.default_rng(seed).permutation(n).astype(np.int32) if shuffle else np.arange(n, dtype=np.int32)
    _check_symbolic(A, perm)


@pytest.mark.slow
@pytest.mark.parametrize("name", ["c2", "c4", "c5"])
def test_symbolic_full_configs(name):
    c = G.CONFIGS[name]
    A, p = G.make_config(c["kind"], c["N"])
    _check_symbolic(A, p)


def test_invalid_arguments():
    A, p = grid("5pt", (8, 8, 1))
    S = mf.Solver(host_only=True)
    with pytest.raises(mf.MfError) as e:
        S.analyze(A.n, A.colptr, A.rowind, np.zeros(A.n, dtype=np.int32))
    assert e.value.code == mf.MF_ERR_ARG
    bad = A.rowind.copy()
    bad[0] = A.n
    with pytest.raises(mf.MfError):
        S.analyze(A.n, A.colptr, bad, p)
    badp = A.colptr.copy()
    badp[3] = badp[4] + 1
    with pytest.raises(mf.MfError):
        S.analyze(A.n, badp, A.rowind, p)
    # host-only contexts refuse numeric work (no CPU fallback)
    S.analyze(A.n, A.colptr, A.rowind, p)
    with pytest.raises(mf.MfError) as e:
        S.factor(A.values)
    assert e.value.code == mf.MF_ERR_STATE


def test_plan_memory_is_planned():
    A, p = grid("27pt", (20, 20, 20))
    inf = _check_symbolic(A, p)
    assert inf["panel_words"] >= inf["nnzL_stored"]
    assert inf["nlevels"] >= 1 and inf["max_front"] > 128


def test_symbolic_postorder_hand_worked():
    """The hand-worked non-postordered etree (tests/golden/postorder_example.json):
    the product's symbolic layer relabels by the same DFS postorder."""
    import json
    from tests.test_oracle_symbolic import _postorder_case
    e = json.load(open(os.path.join(ROOT, "tests", "golden", "postorder_example.json")))
    S = mf.Solver(host_only=True)
    A = _postorder_case(e)
    S.analyze(A.n, A.colptr, A.rowind, np.arange(e["n"], dtype=np.int32))
    np.testing.assert_array_equal(S.perm(), e["final_perm"])
    np.testing.assert_array_equal(S.etree()[0], e["parent_final"])
    q = np.array(e["relabel_q"], dtype=np.int32)
    Aq = _postorder_case(e, q)
    S.analyze(Aq.n, Aq.colptr, Aq.rowind, q)
    np.testing.assert_array_equal(S.perm(), e["final_perm_with_q"])
    _check_symbolic(Aq, q)


@pytest.mark.parametrize("kind,dims", [("27pt", (12, 11, 10)), ("5pt", (40, 30, 1)), ("elast", (6, 6, 6))])
def test_null_perm_library_ordering(kind, dims):
    """perm == NULL: the library orders A itself (METIS nested dissection,
    include/mf.h; reading C4).  The returned final perm is a permutation, the same
    on every call, and the symbolic analysis under it matches the oracle's
    bit-exactly; its fill is in the range of the geometric ND order."""
    A, p = grid(kind, dims)
    S = mf.Solver(host_only=True)
    S.analyze(A.n, A.colptr, A.rowind, None)
    fp = S.perm()
    assert np.array_equal(np.sort(fp), np.arange(A.n))
    S2 = mf.Solver(host_only=True)
    S2.analyze(A.n, A.colptr, A.rowind, None)
    np.testing.assert_array_equal(S2.perm(), fp)
    _check_symbolic(A, fp)          # the final perm is already postordered: analysis is identical
    np.testing.assert_array_equal(S.etree()[0], oracle.symbolic(A, fp).parent)
    Sg = mf.Solver(host_only=True)
    Sg.analyze(A.n, A.colptr, A.rowind, p)
    assert S.info()["flops_true"] <= 2 * Sg.info()["flops_true"]


def test_export_csc_structure_host_only():
    """mf_export_L (supernodal CSC): column j of supernode s holds R_s[jj..f), so
    Lp[n] = nnzL_stored and the row lists are the oracle's (Lx needs a factor)."""
    A, p = grid("27pt", (9, 8, 7))
    S = mf.Solver(host_only=True)
    S.analyze(A.n, A.colptr, A.rowind, p)
    Lp, Li, _ = S.export_L(values=False)
    so = oracle.symbolic(A, p, keep_struct=True)
    assert Lp[-1] == S.info()["nnzL_stored"] == so.stored_L
    for s in range(so.nsuper):
        R = so.rows(s)
        for jj in range(so.k(s)):
            j = int(so.sn_first[s]) + jj
            np.testing.assert_array_equal(Li[Lp[j]:Lp[j + 1]], R[jj:])
            # the true structure of column j is a subset (the rest is padding)
            assert set(so.Li[so.Lp[j]:so.Lp[j + 1]].tolist()) <= set(R[jj:].tolist())


def test_alloc_hooks_must_come_in_pairs():
    o = mf.Options()
    mf.lib.mf_default_options(ctypes.byref(o))
    o.host_only = 1
    keep = mf.DEV_ALLOC_FN(lambda n, u: None)
    o.dev_alloc = ctypes.cast(keep, ctypes.c_void_p)
    h = ctypes.c_void_p()
    assert mf.lib.mf_create(ctypes.byref(h), ctypes.byref(o)) == mf.MF_ERR_ARG
