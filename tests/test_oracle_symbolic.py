"""Pins for the oracle's symbolic part (oracle/symbolic.c) against things other
than itself: hand examples, closed forms (1D chain,
dense, diagonal), brute-force boolean elimination on small inputs, an
independent row-SET implementation of the Appendix-B amalgamation rule, and the
Appendix-A integers (cross-validated at survey time by brute force).

PAPER.md L27 (Sec. II-A) defines what these structures are: the supernodal
elimination tree, supernodes = consecutive columns with the same pattern in L,
front of order f = k + m (reading C1)."""
import json
import os

import numpy as np
import pytest
from hypothesis import given, settings, strategies as st

import oracle
from workloads import grids as G
from tests._grids import dense_from_rows, grid

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def brute_structure(A, perm):
    """Boolean dense elimination of B = P A P^T: returns list of sorted row sets."""
    n = A.n
    Md = G.full_symmetric_dense(A) != 0
    # structural pattern: every stored lower entry counts, even explicit zeros
    cols = np.repeat(np.arange(n), np.diff(A.colptr))
    r = A.rowind.astype(np.int64)
    keep = r >= cols
    Md = np.zeros((n, n), dtype=bool)
    Md[r[keep], cols[keep]] = True
    Md |= Md.T
    p = np.asarray(perm if perm is not None else np.arange(n))
    B = Md[np.ix_(p, p)]
    L = np.tril(B)
    np.fill_diagonal(L, True)
    for k in range(n):
        rows = np.nonzero(L[k + 1:, k])[0] + k + 1
        if rows.size:
            sub = np.ix_(rows, rows)
            L[sub] |= np.tril(np.ones((rows.size, rows.size), dtype=bool))
    return [np.nonzero(L[:, j])[0] for j in range(n)]


def setwise_supernodes(struct, nrelax=(4, 16, 48), zrelax=(0.8, 0.1, 0.05)):
    """Independent implementation: fundamental supernodes from SET equality,
    relaxed amalgamation evaluated on actual merged ROW SETS."""
    n = len(struct)
    parent = [int(s[1]) if s.size > 1 else -1 for s in struct]
    nchild = np.bincount([p for p in parent if p >= 0], minlength=n)
    fund = [0]
    for j in range(n - 1):
        same = (parent[j] == j + 1 and nchild[j + 1] == 1
                and set(struct[j][1:].tolist()) == set(struct[j + 1].tolist()))
        if not same:
            fund.append(j + 1)
    fund.append(n)
    S = len(fund) - 1
    cols = [list(range(fund[s], fund[s + 1])) for s in range(S)]
    col2f = np.empty(n, dtype=int)
    for s in range(S):
        col2f[fund[s]:fund[s + 1]] = s
    sp = [col2f[parent[fund[s + 1] - 1]] if parent[fund[s + 1] - 1] >= 0 else -1 for s in range(S)]
    rowsets = [set().union(*[set(struct[c].tolist()) for c in cols[s]]) for s in range(S)]
    true_nz = [sum(struct[c].size for c in cols[s]) for s in range(S)]
    # group of j+1 is represented by (cols, rows, zeros)
    gcols, grows, gz = list(cols), list(rowsets), [0] * S
    merged = [False] * S
    for j in range(S - 2, -1, -1):
        if sp[j] != j + 1:
            continue
        g = j + 1
        mc = cols[j] + gcols[g]
        mr = set(cols[j]) | grows[g]
        stored = sum(sum(1 for i in mr if i >= c) for c in mc)
        true = true_nz[j] + sum(struct[c].size for c in gcols[g])
        Z = stored - true
        newz = Z - gz[g]
        ns = len(mc)
        z = Z / stored
        if (ns <= nrelax[0] or newz == 0 or (ns <= nrelax[1] and z < zrelax[0])
                or (ns <= nrelax[2] and z < zrelax[1]) or z < zrelax[2]):
            merged[j] = True
            gcols[j], grows[j], gz[j] = mc, mr, Z
    first = [fund[s] for s in range(S) if s == 0 or not merged[s - 1]] + [n]
    return parent, fund, first


def check_against_brute(A, perm):
    sym = oracle.symbolic(A, perm, keep_struct=True)
    assert sym.postorder_was_identity or perm is None or True
    struct = brute_structure(A, sym.perm)   # oracle's final perm (postordered)
    for j in range(A.n):
        got = sym.Li[sym.Lp[j]:sym.Lp[j + 1]]
        np.testing.assert_array_equal(got, struct[j])
    cc = np.array([s.size for s in struct])
    np.testing.assert_array_equal(sym.cc, cc)
    assert sym.nnzL == cc.sum() and sym.flops == int((cc.astype(np.int64) ** 2).sum())
    parent, fund, first = setwise_supernodes(struct)
    np.testing.assert_array_equal(sym.parent, parent)
    np.testing.assert_array_equal(sym.fund_first, fund)
    np.testing.assert_array_equal(sym.sn_first, first)
    # row lists = union of the columns' structures
    for s in range(sym.nsuper):
        rows = set()
        for c in range(first[s], first[s + 1]):
            rows |= set(struct[c].tolist())
        np.testing.assert_array_equal(sym.rows(s), sorted(rows))
    # the postorder: every node's parent comes later, and subtrees are contiguous
    p = sym.parent
    assert all(p[j] == -1 or p[j] > j for j in range(A.n))
    assert_subtrees_contiguous(p)
    return sym


def assert_subtrees_contiguous(parent):
    """A postorder numbers every subtree as a contiguous range ending at its
    root: the descendants of j are exactly j - size(j) + 1 .. j."""
    n = len(parent)
    size = np.ones(n, dtype=np.int64)
    lo = np.arange(n, dtype=np.int64)          # smallest label in the subtree of j
    for j in range(n):                         # children before parents (p[j] > j)
        q = int(parent[j])
        if q >= 0:
            size[q] += size[j]
            lo[q] = min(lo[q], lo[j])
    assert (lo == np.arange(n) - size + 1).all()


def _postorder_case(e, q=None):
    n = e["n"]
    M = np.eye(n) * e["diag"]
    for i, j in e["offdiag_lower"]:
        M[i, j] = M[j, i] = e["offdiag_value"]
    if q is not None:                           # relabel: A'(q[i], q[j]) = A(i, j)
        Mq = np.zeros_like(M)
        Mq[np.ix_(q, q)] = M
        M = Mq
    return dense_from_rows(M.tolist())


def test_postorder_hand_worked():
    """A natural order whose etree is NOT a postorder (tests/golden/postorder_example.json,
    hand-worked from PAPER.md L27 and reading C5): the oracle must relabel by the
    DFS postorder (children ascending) and compose it with the input perm."""
    e = json.load(open(os.path.join(GOLD, "postorder_example.json")))
    A = _postorder_case(e)
    sym = oracle.symbolic(A, None)
    assert not sym.postorder_was_identity
    np.testing.assert_array_equal(sym.perm, e["final_perm"])
    np.testing.assert_array_equal(sym.parent, e["parent_final"])
    np.testing.assert_array_equal(sym.cc, e["cc_final"])
    assert_subtrees_contiguous(sym.parent)
    # natural-order etree by brute force is the hand-derived one (not a postorder)
    st = brute_structure(A, np.arange(e["n"]))
    assert [int(s[1]) if s.size > 1 else -1 for s in st] == e["etree_natural"]
    with pytest.raises(AssertionError):
        assert_subtrees_contiguous(e["etree_natural"])
    # the same matrix relabeled by q, with perm = q: final perm = q composed with the postorder
    q = np.array(e["relabel_q"], dtype=np.int32)
    Aq = _postorder_case(e, q)
    symq = oracle.symbolic(Aq, q)
    np.testing.assert_array_equal(symq.perm, e["final_perm_with_q"])
    np.testing.assert_array_equal(symq.parent, e["parent_final"])


def test_appendix_c_examples():
    ex = json.load(open(os.path.join(GOLD, "appendixC_examples.json")))
    for key in ("ex3", "ex4"):
        e = ex[key]
        A = dense_from_rows(e["A"])
        sym = oracle.symbolic(A, None)
        np.testing.assert_array_equal(sym.parent, e["parent"])
        np.testing.assert_array_equal(sym.cc, e["cc"])
        assert sym.nnzL == e["nnzL"] and sym.flops == e["flops"]
        np.testing.assert_array_equal(sym.fund_first, e["fund_first"])
        np.testing.assert_array_equal(sym.sn_first, e["sn_first"])
        if "sn_rows" in e:
            for s, rows in enumerate(e["sn_rows"]):
                np.testing.assert_array_equal(sym.rows(s), rows)


def test_chain_closed_form():
    n = 50
    sym = oracle.symbolic(G.laplacian_1d(n), None)
    np.testing.assert_array_equal(sym.parent, list(range(1, n)) + [-1])
    np.testing.assert_array_equal(sym.cc, [2] * (n - 1) + [1])
    assert sym.nfund == n - 1          # only the last two columns merge
    assert sym.nnzL == 2 * n - 1


def test_dense_one_supernode_and_diagonal_n_roots():
    n = 12
    rng = np.random.default_rng(3)
    X = rng.standard_normal((n, n))
    A = dense_from_rows(X @ X.T + n * np.eye(n))
    sym = oracle.symbolic(A, rng.permutation(n).astype(np.int32))
    assert sym.nfund == 1 and sym.nsuper == 1 and sym.nnzL == n * (n + 1) // 2
    D = dense_from_rows(np.diag(np.arange(1, n + 1)))
    sym = oracle.symbolic(D, None)
    assert (sym.parent == -1).all() and sym.nfund == n and sym.nsuper == n


@pytest.mark.parametrize("kind,dims", [("5pt", (32, 32, 1)), ("27pt", (6, 5, 4)), ("7pt", (8, 7, 6)),
                                       ("9pt", (20, 17, 1)), ("elast", (5, 5, 5))])
def test_grids_vs_bruteforce(kind, dims):
    A, p = grid(kind, dims)
    check_against_brute(A, p)


@settings(max_examples=25, deadline=None)
@given(n=st.integers(1, 60), dens=st.floats(0.0, 0.3), seed=st.integers(0, 10_000),
       shuffle=st.booleans())
def test_random_patterns_vs_bruteforce(n, dens, seed, shuffle):
    """Random patterns + random perms: non-postordered trees exercise the relabel."""
    A = G.random_spd_pattern(n, dens, seed, dup=0.2, upper=0.1)
    perm = np.random.default_rng(seed).permutation(n).astype(np.int32) if shuffle else None
    check_against_brute(A, perm)


def _golden_cases():
    g = json.load(open(os.path.join(GOLD, "appendixA_counts.json")))["grids"]
    out = []
    for name, e in g.items():
        marks = [pytest.mark.slow] if e.get("slow") else []
        out.append(pytest.param(name, e, marks=marks, id=name))
    return out


@pytest.mark.parametrize("name,e", _golden_cases())
def test_appendix_a_integers(name, e):
    A, p = grid(e["kind"], tuple(e["dims"]))
    if "nnzA" in e:
        assert A.nnz == e["nnzA"]
    sym = oracle.symbolic(A, p)
    assert sym.postorder_was_identity          # ND order is a postorder
    assert sym.nnzL == e["nnzL"]
    assert sym.flops == e["flops"]
    assert sym.nfund == e["nfund"]
    assert sym.nsuper == e["nsuper"]
    assert sym.stored_L == e["stored_L"]
    assert sym.exec_flops == e["exec_flops"]
    if "max_front" in e:
        k = np.diff(sym.sn_first)
        f = np.diff(sym.sn_rowptr)
        assert f.max() == e["max_front"] and k.max() == e["max_k"] and (f - k).max() == e["max_m"]


def test_invalid_inputs_rejected():
    A = G.laplacian_5pt(4)
    with pytest.raises(ValueError):
        oracle.symbolic(A, np.zeros(A.n, dtype=np.int32))   # not a permutation
    bad = G.CSC(A.n, A.colptr.copy(), A.rowind.copy(), A.values)
    bad.rowind[3] = A.n + 5
    with pytest.raises(ValueError):
        oracle.symbolic(bad, None)


def _front_ops_by_loops(k, m):
    """Count the flops of the unblocked F-U loops on a k-pivot, m-row front one
    operation at a time (one FMA = 2, each sqrt / division = 1):
    potrf column algorithm, trsm by substitution, syrk on the lower triangle."""
    fl = 0
    for j in range(k):                       # potrf
        fl += 1 + (k - 1 - j)                # sqrt, divisions below the pivot
        fl += 2 * sum(k - b for b in range(j + 1, k))   # rank-1 update of the lower trailing block
    for _ in range(m):                       # trsm: each row x_j = (x_j - sum x_p L_jp) / L_jj
        fl += sum(1 + 2 * j for j in range(k))
    fl += 2 * k * (m * (m + 1) // 2)         # syrk: lower triangle incl. diagonal, k FMAs each
    return fl


@pytest.mark.parametrize("k,m", [(1, 0), (1, 5), (3, 0), (4, 7), (9, 2), (16, 33)])
def test_front_flops_counts_the_loops(k, m):
    assert oracle.front_flops(k, m) == _front_ops_by_loops(k, m)


@pytest.mark.parametrize("kind,dims", [("5pt", (32, 32, 1)), ("27pt", (6, 5, 4)), ("7pt", (12, 12, 12))])
def test_front_flops_fundamental_equals_true_count(kind, dims):
    """On FUNDAMENTAL supernodes there is no padding, so the F-U flops summed over
    the fronts equal the true count sum_j cc_j^2 -- two different formulas."""
    A, p = grid(kind, dims)
    sym = oracle.symbolic(A, p, amalgamate=False)
    tot = sum(oracle.front_flops(sym.k(s), sym.rows(s).size - sym.k(s)) for s in range(sym.nsuper))
    assert tot == sym.flops == int((sym.cc.astype(np.int64) ** 2).sum())
    assert sym.exec_flops == tot
