"""Exchange callbacks for multi-GPU factorizations (include/mf.h, mf_set_exchange).

The library decides WHAT moves (the update matrices of the subtree roots, the
solve vectors); these callbacks only move bytes between device buffers:

* ``TorchDistExchange`` -- NCCL over NVLink through ``torch.distributed`` (one
  process per GPU): batched isend/irecv, broadcast, all-reduce.
* ``LoopbackHub`` -- P virtual ranks inside ONE process on one GPU (threads),
  used by the tests to run the multi-rank code path without a multi-GPU box.
"""
from __future__ import annotations

import threading

import torch

from .mf import MF_XFER_ALLREDUCE_MIN_I32, MF_XFER_ALLREDUCE_SUM, MF_XFER_BCAST, MF_XFER_RECV, MF_XFER_SEND


class _DevBuf:
    """A raw device pointer seen as a 1-D CUDA array (no copy)."""

    def __init__(self, ptr: int, nbytes: int, typestr: str):
        itemsize = 4 if typestr == "<i4" else 8
        self.__cuda_array_interface__ = {"shape": (nbytes // itemsize,), "typestr": typestr,
                                         "data": (ptr, False), "version": 3, "strides": None}


def device_tensor(ptr: int, nbytes: int, int32: bool = False) -> torch.Tensor:
    return torch.as_tensor(_DevBuf(ptr, nbytes, "<i4" if int32 else "<f8"), device="cuda")


def host_tensor(ptr: int, nbytes: int, int32: bool = False) -> torch.Tensor:
    """A raw HOST pointer as a tensor (no copy) -- for exercising the exchange
    logic with the gloo backend on CPU-only hosts."""
    import ctypes
    import numpy as np
    ct = ctypes.c_int32 if int32 else ctypes.c_double
    n = nbytes // ctypes.sizeof(ct)
    arr = np.ctypeslib.as_array(ctypes.cast(ptr, ctypes.POINTER(ct)), shape=(n,))
    return torch.from_numpy(arr)


class TorchDistExchange:
    """NCCL collectives/point-to-point through the default torch.distributed group.
    ``host=True``: the pointers are host memory (gloo tests on CPU).
    ``stage=True``: the pointers are device memory but the group's backend cannot
    touch it (gloo): every buffer is staged through a host copy -- lets several
    ranks share ONE GPU in tests (NCCL refuses two ranks on one device)."""

    def __init__(self, host: bool = False, stage: bool = False):
        self.view = host_tensor if host else device_tensor
        self.host = host
        self.stage = stage and not host
        self._first = True

    def __call__(self, ops):
        import torch.distributed as dist
        if self._first:   # every rank reaches the first exchange: create the communicator collectively
            dist.barrier()
            self._first = False
        view = self.view
        if self.stage:   # device buffers through host copies (gloo), written back after the transfers
            torch.cuda.synchronize()
            staged = []

            def view(ptr, nbytes, int32=False, _dev=device_tensor):
                d = _dev(ptr, nbytes, int32=int32)
                h = d.cpu()
                staged.append((d, h))
                return h
        p2p = []
        for op, peer, ptr, nbytes in ops:
            if op in (MF_XFER_SEND, MF_XFER_RECV):
                t = view(ptr, nbytes)
                p2p.append(dist.P2POp(dist.isend if op == MF_XFER_SEND else dist.irecv, t, peer))
        if p2p:
            for req in dist.batch_isend_irecv(p2p):
                req.wait()
        for op, peer, ptr, nbytes in ops:
            if op == MF_XFER_BCAST:
                dist.broadcast(view(ptr, nbytes), src=peer)
            elif op == MF_XFER_ALLREDUCE_SUM:
                dist.all_reduce(view(ptr, nbytes))
            elif op == MF_XFER_ALLREDUCE_MIN_I32:
                dist.all_reduce(view(ptr, nbytes, int32=True), op=dist.ReduceOp.MIN)
        if self.stage:
            for d, h in staged:
                d.copy_(h)
        if not self.host:
            torch.cuda.synchronize()


class LoopbackHub:
    """P virtual ranks in one process (one thread each); the transfers are device copies."""

    def __init__(self, nranks: int):
        self.nranks = nranks
        self.ops = [None] * nranks
        self.barrier = threading.Barrier(nranks)
        self.error = None

    def for_rank(self, rank: int):
        def fn(ops):
            self.ops[rank] = list(ops)
            self.barrier.wait()
            if rank == 0:
                try:
                    self._execute()
                except Exception as e:  # noqa: BLE001
                    self.error = e
            self.barrier.wait()
            if self.error is not None:
                raise RuntimeError(f"loopback exchange failed: {self.error}")
        return fn

    def _execute(self):
        torch.cuda.synchronize()
        R = self.nranks
        # point-to-point: match the k-th send r -> p with the k-th receive on p from r
        sends = {(r, op[1]): [] for r in range(R) for op in self.ops[r] if op[0] == MF_XFER_SEND}
        for r in range(R):
            for op in self.ops[r]:
                if op[0] == MF_XFER_SEND:
                    sends[(r, op[1])].append(op)
        for p in range(R):
            cnt = {}
            for op in self.ops[p]:
                if op[0] != MF_XFER_RECV:
                    continue
                src = op[1]
                i = cnt.get(src, 0)
                cnt[src] = i + 1
                s = sends[(src, p)][i]
                assert s[3] == op[3], "send/recv size mismatch"
                device_tensor(op[2], op[3]).copy_(device_tensor(s[2], s[3]))
        # collectives: the k-th collective of every rank form one group
        colls = [[op for op in self.ops[r] if op[0] in (MF_XFER_BCAST, MF_XFER_ALLREDUCE_SUM,
                                                        MF_XFER_ALLREDUCE_MIN_I32)] for r in range(R)]
        for k in range(len(colls[0])):
            group = [colls[r][k] for r in range(R)]
            kind = group[0][0]
            assert all(g[0] == kind and g[3] == group[0][3] for g in group)
            i32 = kind == MF_XFER_ALLREDUCE_MIN_I32
            ts = [device_tensor(g[2], g[3], int32=i32) for g in group]
            if kind == MF_XFER_BCAST:
                root = ts[group[0][1]]
                for t in ts:
                    if t.data_ptr() != root.data_ptr():
                        t.copy_(root)
            elif kind == MF_XFER_ALLREDUCE_SUM:
                acc = ts[0].clone()
                for t in ts[1:]:
                    acc += t
                for t in ts:
                    t.copy_(acc)
            else:
                acc = ts[0].clone()
                for t in ts[1:]:
                    acc = torch.minimum(acc, t)
                for t in ts:
                    t.copy_(acc)
        torch.cuda.synchronize()
