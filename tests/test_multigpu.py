"""Multi-GPU path: subtree-to-GPU mapping, broadcast of the
frontier roots' update matrices, every rank holds the top supernodes and factors
the large ones cooperatively (block-cyclic pivot-column blocks broadcast by their
owner, trailing updates split by owned column, U^n all-gathered).

CPU (not gpu): the mapping is a partition consistent across ranks (checked in
two gloo processes, world size 2), and the exchange callback moves the right
bytes (TorchDistExchange over gloo with host buffers).
GPU: P virtual ranks on one GPU (LoopbackHub, one thread per rank) reproduce
the single-rank factor (bit-exactly on manufactured inputs) and the solve."""
import os
import threading

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import paper_conf_ipps_georgesgsc11_b200 as mf
from paper_conf_ipps_georgesgsc11_b200 import mf as mfmod
from tests._grids import grid


def mapping_for(A, p, R, rank, split_all=True):
    S = mf.Solver(host_only=True, nranks=R, rank=rank, split_all=split_all)
    S.analyze(A.n, A.colptr, A.rowind, p)
    owner, top, load, top_load = S.mapping()
    sn = S.supernodes()
    inf = S.info()
    S.close()
    return owner, top, load, top_load, sn, inf


@pytest.mark.parametrize("split_all", [True, False])
@pytest.mark.parametrize("R", [2, 3, 4, 8])
@pytest.mark.parametrize("kind,dims", [("27pt", (20, 20, 20)), ("9pt", (60, 60, 1)), ("elast", (8, 8, 8))])
def test_mapping_is_a_partition(kind, dims, R, split_all):
    A, p = grid(kind, dims)
    owner, top, load, top_load, sn, inf = mapping_for(A, p, R, 0, split_all)
    if split_all:   # forced split: at least R subtrees below the top
        assert top.any() and len(set(owner[~top])) == R
    par = sn["sn_parent"]
    ns = inf["nsuper"]
    # top is closed upward; below the frontier every supernode has its subtree's owner
    for s in range(ns):
        if top[s] and par[s] >= 0:
            assert top[par[s]]
        if not top[s] and par[s] >= 0 and not top[par[s]]:
            assert owner[s] == owner[par[s]]
    assert set(owner[~top]) <= set(range(R))
    k = np.diff(sn["sn_first"]).astype(float)
    f = np.diff(sn["sn_rowptr"]).astype(float)
    m = f - k
    fl = k * m * m + m * k * (k + 1) + k * (k + 1) * (2 * k + 1) / 6
    assert load.sum() + top_load == pytest.approx(fl.sum(), rel=1e-12)
    assert top_load == pytest.approx(fl[top].sum(), rel=1e-12)
    for r in range(R):
        assert load[r] == pytest.approx(fl[(~top) & (owner == r)].sum(), rel=1e-12)
    # every rank computes the same mapping
    for r in range(1, R):
        o2, t2, l2, tl2, _, _ = mapping_for(A, p, R, r, split_all)
        np.testing.assert_array_equal(o2, owner)
        np.testing.assert_array_equal(t2, top)


def _gloo_worker(rank, world, port, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        A, p = grid("27pt", (16, 16, 16))
        owner, top, load, top_load, sn, inf = mapping_for(A, p, world, rank)
        # all ranks agree on the mapping
        t = torch.from_numpy(owner.astype(np.int64))
        gathered = [torch.empty_like(t) for _ in range(world)]
        dist.all_gather(gathered, t)
        same = all(torch.equal(g, gathered[0]) for g in gathered)
        # exchange semantics over gloo with host buffers: rank r sends its buffer to 0,
        # then broadcast and the two reductions
        from paper_conf_ipps_georgesgsc11_b200.exchange import TorchDistExchange
        ex = TorchDistExchange(host=True)
        bufs = [np.full(5, float(r + 1)) for r in range(world)]
        ops = []
        if rank == 0:
            for r in range(1, world):
                ops.append((mfmod.MF_XFER_RECV, r, bufs[r].ctypes.data, bufs[r].nbytes))
        else:
            ops.append((mfmod.MF_XFER_SEND, 0, bufs[rank].ctypes.data, bufs[rank].nbytes))
        own = np.full(3, float(rank + 1))
        bc = np.full(4, float(rank + 10))
        mn = np.array([rank + 7], dtype=np.int32)
        ops += [(mfmod.MF_XFER_ALLREDUCE_SUM, 0, own.ctypes.data, own.nbytes),
                (mfmod.MF_XFER_BCAST, 0, bc.ctypes.data, bc.nbytes),
                (mfmod.MF_XFER_ALLREDUCE_MIN_I32, 0, mn.ctypes.data, mn.nbytes)]
        ex(ops)
        ok = same
        if rank == 0:
            ok = ok and all((bufs[r] == r + 1).all() for r in range(world))
        ok = ok and (own == world * (world + 1) / 2).all() and (bc == 10.0).all() and mn[0] == 7
        q.put((rank, bool(ok)))
    finally:
        dist.destroy_process_group()


def test_gloo_world2_mapping_and_exchange():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = 29500 + os.getpid() % 1000
    procs = [ctx.Process(target=_gloo_worker, args=(r, 2, port, q)) for r in range(2)]
    for pr in procs:
        pr.start()
    res = dict(q.get(timeout=300) for _ in procs)
    for pr in procs:
        pr.join(timeout=60)
    assert res == {0: True, 1: True}


# ---------------------------------------------------------------- GPU (loopback ranks)
def run_loopback(A, perm, R, values=None, b=None, split_all=True, junk_others=True, profiling=0, **opts):
    from paper_conf_ipps_georgesgsc11_b200.exchange import LoopbackHub
    hub = LoopbackHub(R)
    solvers = [mf.Solver(nranks=R, rank=r, exchange=hub.for_rank(r), split_all=split_all, **opts) for r in range(R)]
    for S in solvers:
        S.analyze(A.n, A.colptr, A.rowind, perm)
        if profiling:
            S.set_profiling(profiling)
    vals = A.values if values is None else values
    errs = [None] * R
    xs = [None] * R

    def work(r):
        try:
            # only rank 0's values / b are read (include/mf.h): the others pass junk
            solvers[r].factor(vals if r == 0 or not junk_others else np.full_like(vals, np.nan))
            if b is not None:
                xs[r] = solvers[r].solve(b if r == 0 or not junk_others else np.zeros_like(b))
        except Exception as e:  # noqa: BLE001
            errs[r] = e
    th = [threading.Thread(target=work, args=(r,)) for r in range(R)]
    for t in th:
        t.start()
    for t in th:
        t.join(timeout=600)
    assert all(e is None for e in errs), errs
    return solvers, xs


LOOPBACK_CASES = [("27pt", (20, 20, 20), {}), ("7pt", (24, 24, 24), {}),
                  ("27pt", (20, 20, 20), {"panel_w": 16}), ("27pt", (32, 32, 32), {})]


@pytest.mark.gpu
@pytest.mark.parametrize("R", [2, 3, 4])
@pytest.mark.parametrize("kind,dims,opts", LOOPBACK_CASES)
def test_loopback_ranks_match_single(kind, dims, opts, R):
    from tests.test_gpu_parity import c11, spmv, backward_error
    from workloads import grids as G
    A, p = grid(kind, dims)
    ref = mf.Solver(**opts)
    ref.analyze(A.n, A.colptr, A.rowind, p)
    ref.factor(A.values)
    b = spmv(A, G.rhs(A.n, 0))
    xref = ref.solve(b)
    solvers, xs = run_loopback(A, p, R, b=b, **opts)
    owner, top, load, _ = solvers[0].mapping()
    coop = solvers[0].cooperative()
    assert top.any() and len(set(owner[~top])) == R
    if opts or dims[0] >= 32:   # cases with fronts wide enough to be shared
        assert coop.any()
    sn = ref.supernodes()
    worst = 0.0
    for s in range(ref.info()["nsuper"]):
        f = int(sn["sn_rowptr"][s + 1] - sn["sn_rowptr"][s])
        k = int(sn["sn_first"][s + 1] - sn["sn_first"][s])
        holders = range(R) if top[s] else [int(owner[s])]   # the top is replicated on every rank
        for r in holders:
            worst = max(worst, c11(solvers[r].panel(s, f, k), ref.panel(s, f, k)))
    assert worst <= 1e-12
    for r in range(R):
        np.testing.assert_allclose(xs[r], xref, rtol=1e-11, atol=1e-13)
        assert backward_error(A, xs[r], b) <= 1e-12
    for r in range(1, R):
        np.testing.assert_array_equal(xs[r], xs[0])


@pytest.mark.gpu
@pytest.mark.parametrize("R", [2, 3, 4])
@pytest.mark.parametrize("dims,opts", [((12, 12, 12), {}), ((16, 16, 16), {"panel_w": 16})])
def test_loopback_manufactured_bit_exact(R, dims, opts):
    """SURVEY.md Sec. 8(c) 'Multi-GPU' pin: the manufactured factor is reproduced
    bitwise by every rank, whatever the split of the top fronts' work."""
    import oracle
    from workloads import grids as G
    A0, p = grid("27pt", dims)
    s0 = oracle.symbolic(A0, p, keep_struct=True)
    A, Lx = G.manufactured(A0.n, s0.Lp, s0.Li, s0.perm, seed=1234)
    ref = mf.Solver(**opts)
    ref.analyze(A.n, A.colptr, A.rowind, s0.perm)
    ref.factor(A.values)
    solvers, _ = run_loopback(A, s0.perm, R, **opts)
    owner, top, _, _ = solvers[0].mapping()
    if opts:
        assert solvers[0].cooperative().any()
    sn = ref.supernodes()
    for s in range(ref.info()["nsuper"]):
        f = int(sn["sn_rowptr"][s + 1] - sn["sn_rowptr"][s])
        k = int(sn["sn_first"][s + 1] - sn["sn_first"][s])
        for r in (range(R) if top[s] else [int(owner[s])]):
            np.testing.assert_array_equal(solvers[r].panel(s, f, k), ref.panel(s, f, k))


@pytest.mark.gpu
@pytest.mark.parametrize("profiling", [1, 2])
def test_loopback_profiling_modes(profiling):
    """Per-launch timing on P ranks (the top program's segments between exchange
    points always run eagerly with events) leaves the factor bitwise unchanged; in
    timeline mode every rank's local program has a timeline."""
    import oracle
    from workloads import grids as G
    A0, p = grid("27pt", (12, 12, 12))
    s0 = oracle.symbolic(A0, p, keep_struct=True)
    A, Lx = G.manufactured(A0.n, s0.Lp, s0.Li, s0.perm, seed=1234)
    ref = mf.Solver()
    ref.analyze(A.n, A.colptr, A.rowind, s0.perm)
    ref.factor(A.values)
    R = 2
    solvers, _ = run_loopback(A, s0.perm, R, profiling=profiling, panel_w=16)
    owner, top, _, _ = solvers[0].mapping()
    sn = ref.supernodes()
    for s in range(ref.info()["nsuper"]):
        f = int(sn["sn_rowptr"][s + 1] - sn["sn_rowptr"][s])
        k = int(sn["sn_first"][s + 1] - sn["sn_first"][s])
        for r in (range(R) if top[s] else [int(owner[s])]):
            np.testing.assert_array_equal(solvers[r].panel(s, f, k), ref.panel(s, f, k))
    for S in solvers:
        assert sum(k["launches"] for k in S.kernel_stats()) > 0
        if profiling == 2:
            t0, t1 = S.launch_timeline()
            assert (t1 >= t0).all()


@pytest.mark.gpu
def test_loopback_not_spd_reported_on_every_rank():
    from workloads import grids as G
    A, p = grid("27pt", (14, 14, 14))
    v = A.values.copy()
    victim = int(p[-1])   # a top column (last in the order)
    d = A.colptr[victim] + np.nonzero(A.rowind[A.colptr[victim]:A.colptr[victim + 1]] == victim)[0][0]
    v[d] = -100.0
    from paper_conf_ipps_georgesgsc11_b200.exchange import LoopbackHub
    R = 3
    hub = LoopbackHub(R)
    solvers = [mf.Solver(nranks=R, rank=r, exchange=hub.for_rank(r), split_all=True) for r in range(R)]
    for S in solvers:
        S.analyze(A.n, A.colptr, A.rowind, p)
    cols = [None] * R

    def work(r):
        try:
            solvers[r].factor(v)
        except mf.MfNotSPD as e:
            cols[r] = e.failed_col
    th = [threading.Thread(target=work, args=(r,)) for r in range(R)]
    for t in th:
        t.start()
    for t in th:
        t.join()
    assert cols == [victim] * R


def _staged_worker(rank, world, port, dims, q):
    """One rank of a real torch.distributed job on ONE GPU: gloo with host staging
    (TorchDistExchange(stage=True)); returns the hashes of its panels."""
    import hashlib
    import oracle
    from workloads import grids as G
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from paper_conf_ipps_georgesgsc11_b200.exchange import TorchDistExchange
        A0, p = grid("27pt", dims)
        s0 = oracle.symbolic(A0, p, keep_struct=True)
        A, _ = G.manufactured(A0.n, s0.Lp, s0.Li, s0.perm, seed=1234)
        S = mf.Solver(nranks=world, rank=rank, exchange=TorchDistExchange(stage=True), split_all=True,
                      panel_w=16)
        S.analyze(A.n, A.colptr, A.rowind, s0.perm)
        # only rank 0's values are read: the others pass NaN
        S.factor(A.values if rank == 0 else np.full_like(A.values, np.nan))
        owner, top, _, _ = S.mapping()
        sn = S.supernodes()
        h = {}
        for s in range(S.info()["nsuper"]):
            if top[s] or owner[s] == rank:
                f = int(sn["sn_rowptr"][s + 1] - sn["sn_rowptr"][s])
                k = int(sn["sn_first"][s + 1] - sn["sn_first"][s])
                h[s] = hashlib.sha256(S.panel(s, f, k).tobytes()).hexdigest()
        b = np.arange(A.n, dtype=np.float64) % 7 - 3.0
        x = S.solve(b if rank == 0 else np.zeros_like(b))
        q.put((rank, h, hashlib.sha256(x.tobytes()).hexdigest(), int(S.cooperative().sum())))
    except Exception as e:  # noqa: BLE001
        import traceback
        q.put((rank, None, traceback.format_exc(), 0))
    finally:
        dist.destroy_process_group()


@pytest.mark.gpu
@pytest.mark.parametrize("dims", [(14, 14, 14), (16, 15, 14)])
def test_torchdist_two_processes_one_gpu_bitwise(dims):
    """the real TorchDistExchange (torch.distributed, here gloo with host
    staging: two processes on one GPU) reproduces the single-rank factor BITWISE on
    manufactured input (SURVEY.md Sec. 8(c) multi-GPU pin), with cooperative top fronts,
    rank 0's values / b broadcast, and the same solve on every rank."""
    import hashlib
    import oracle
    from workloads import grids as G
    A0, p = grid("27pt", dims)
    s0 = oracle.symbolic(A0, p, keep_struct=True)
    A, _ = G.manufactured(A0.n, s0.Lp, s0.Li, s0.perm, seed=1234)
    ref = mf.Solver(panel_w=16)
    ref.analyze(A.n, A.colptr, A.rowind, s0.perm)
    ref.factor(A.values)
    b = np.arange(A.n, dtype=np.float64) % 7 - 3.0
    xref = hashlib.sha256(ref.solve(b).tobytes()).hexdigest()
    sn = ref.supernodes()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = 29700 + os.getpid() % 1000
    procs = [ctx.Process(target=_staged_worker, args=(r, 2, port, dims, q)) for r in range(2)]
    for pr in procs:
        pr.start()
    res = dict((r, (h, x, nc)) for r, h, x, nc in (q.get(timeout=900) for _ in procs))
    for pr in procs:
        pr.join(timeout=120)
    for r in range(2):
        h, x, nc = res[r]
        assert h is not None, x
        assert nc > 0   # cooperative top fronts exercised
        for s, hs in h.items():
            f = int(sn["sn_rowptr"][s + 1] - sn["sn_rowptr"][s])
            k = int(sn["sn_first"][s + 1] - sn["sn_first"][s])
            assert hs == hashlib.sha256(ref.panel(s, f, k).tobytes()).hexdigest(), (r, s)
        assert x == xref, r
