"""ctypes binding of include/mf.h -- argument marshalling only.

Every step of the hot path runs inside libmf.so (CUDA kernels for sm_100a);
this module converts numpy arrays / torch tensors to raw pointers and return
codes to exceptions.  It never computes anything itself and has no fallback.
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

from ._build import LIB as _LIB_PATH

MF_OK = 0
MF_NOT_SPD = 1
MF_ERR_ARG = -1
MF_ERR_STATE = -2
MF_ERR_NOMEM = -3
MF_ERR_CUDA = -4
MF_ERR_NCCL = -5

# every symbol include/mf.h declares (checked by tests/test_abi.py)
EXPORTED_SYMBOLS = (
    "mf_default_options", "mf_create", "mf_analyze", "mf_factor", "mf_solve", "mf_get_info",
    "mf_get_perm", "mf_get_etree", "mf_get_supernodes", "mf_export_panel", "mf_export_diag", "mf_export_L",
    "mf_export_panels", "mf_solve_nrhs",
    "mf_get_program", "mf_set_profiling", "mf_get_kernel_stats", "mf_set_exchange", "mf_get_mapping", "mf_destroy", "mf_strerror",
    "mf_get_launch_times", "mf_get_launch_timeline", "mf_set_variant_model", "mf_get_variants",
)
MF_VARIANTS = 7
MF_VARIANT_FEATURES = 9


class Options(ctypes.Structure):
    _fields_ = [
        ("amalgamate", ctypes.c_int32), ("nrelax", ctypes.c_int32 * 3), ("zrelax", ctypes.c_double * 3),
        ("small_front_max", ctypes.c_int32), ("panel_w", ctypes.c_int32), ("device", ctypes.c_int32),
        ("host_only", ctypes.c_int32), ("nranks", ctypes.c_int32), ("rank", ctypes.c_int32),
        ("stream", ctypes.c_void_p), ("split_all", ctypes.c_int32), ("nbranch", ctypes.c_int32),
        ("fuse_ea", ctypes.c_int32), ("lookahead", ctypes.c_int32),
        ("dev_alloc", ctypes.c_void_p), ("dev_free", ctypes.c_void_p), ("alloc_user", ctypes.c_void_p),
        ("ozaki_slices", ctypes.c_int32), ("refine_iters", ctypes.c_int32),
    ]


DEV_ALLOC_FN = ctypes.CFUNCTYPE(ctypes.c_void_p, ctypes.c_size_t, ctypes.c_void_p)
DEV_FREE_FN = ctypes.CFUNCTYPE(None, ctypes.c_void_p, ctypes.c_void_p)


class Info(ctypes.Structure):
    _fields_ = [
        ("n", ctypes.c_int64), ("nnzA", ctypes.c_int64), ("nnzL", ctypes.c_int64),
        ("nnzL_stored", ctypes.c_int64), ("panel_words", ctypes.c_int64), ("flops_true", ctypes.c_int64),
        ("flops_exec", ctypes.c_int64), ("nfund", ctypes.c_int32), ("nsuper", ctypes.c_int32),
        ("nlevels", ctypes.c_int32), ("max_front", ctypes.c_int32), ("rows_total", ctypes.c_int64),
        ("failed_col", ctypes.c_int64), ("workspace_bytes", ctypes.c_int64), ("launches_factor", ctypes.c_int64),
        ("t_analyze", ctypes.c_double), ("t_factor", ctypes.c_double), ("t_solve", ctypes.c_double),
        ("nbranch", ctypes.c_int32), ("ozaki_slices", ctypes.c_int32), ("refine_steps", ctypes.c_int32),
        ("solve_berr", ctypes.c_double), ("launches_ozaki", ctypes.c_int64),
    ]

    def as_dict(self) -> dict:
        return {k: getattr(self, k) for k, _ in self._fields_}


class KernelStat(ctypes.Structure):
    _fields_ = [("name", ctypes.c_char * 32), ("launches", ctypes.c_int64), ("ms", ctypes.c_double),
                ("flops", ctypes.c_double), ("bytes", ctypes.c_double)]


MF_KERNEL_CLASSES = 7

MF_XFER_SEND, MF_XFER_RECV, MF_XFER_BCAST, MF_XFER_ALLREDUCE_SUM, MF_XFER_ALLREDUCE_MIN_I32 = 1, 2, 3, 4, 5


class Xfer(ctypes.Structure):
    _fields_ = [("op", ctypes.c_int32), ("peer", ctypes.c_int32), ("ptr", ctypes.c_void_p), ("bytes", ctypes.c_int64)]


EXCHANGE_FN = ctypes.CFUNCTYPE(ctypes.c_int, ctypes.c_void_p, ctypes.POINTER(Xfer), ctypes.c_int64)


class LaunchInfo(ctypes.Structure):
    _fields_ = [("kind", ctypes.c_int32), ("level", ctypes.c_int32), ("count", ctypes.c_int64),
                ("flops", ctypes.c_double), ("bytes", ctypes.c_double), ("int8_ops", ctypes.c_double),
                ("stream", ctypes.c_int32), ("reserved", ctypes.c_int32)]


def lib_path() -> str:
    return _LIB_PATH


def _load():
    if not os.path.exists(_LIB_PATH):
        raise ImportError(f"libmf.so not built at {_LIB_PATH}: run `python -c 'import __graft_entry__ as g; g.build()'`"
                          " (there is no CPU fallback)")
    L = ctypes.CDLL(_LIB_PATH)
    vp, i32, i64 = ctypes.c_void_p, ctypes.c_int32, ctypes.c_int64
    sig = {
        "mf_default_options": ([ctypes.POINTER(Options)], ctypes.c_int),
        "mf_create": ([ctypes.POINTER(vp), ctypes.POINTER(Options)], ctypes.c_int),
        "mf_analyze": ([vp, i64, vp, vp, vp], ctypes.c_int),
        "mf_factor": ([vp, vp], ctypes.c_int),
        "mf_solve": ([vp, vp, vp], ctypes.c_int),
        "mf_get_info": ([vp, ctypes.POINTER(Info)], ctypes.c_int),
        "mf_get_perm": ([vp, vp], ctypes.c_int),
        "mf_get_etree": ([vp, vp, vp], ctypes.c_int),
        "mf_get_supernodes": ([vp, vp, vp, vp, vp, vp], ctypes.c_int),
        "mf_export_panel": ([vp, i32, vp], ctypes.c_int),
        "mf_export_diag": ([vp, vp], ctypes.c_int),
        "mf_export_L": ([vp, vp, vp, vp], ctypes.c_int),
        "mf_export_panels": ([vp, vp], ctypes.c_int),
        "mf_solve_nrhs": ([vp, i32, vp, i64, vp, i64], ctypes.c_int),
        "mf_get_program": ([vp, ctypes.POINTER(LaunchInfo), i64, ctypes.POINTER(i64)], ctypes.c_int),
        "mf_set_exchange": ([vp, EXCHANGE_FN, vp], ctypes.c_int),
        "mf_get_mapping": ([vp, vp, vp, vp, vp], ctypes.c_int),
        "mf_set_profiling": ([vp, ctypes.c_int], ctypes.c_int),
        "mf_get_kernel_stats": ([vp, ctypes.POINTER(KernelStat), ctypes.POINTER(i32)], ctypes.c_int),
        "mf_destroy": ([vp], None),
        "mf_strerror": ([ctypes.c_int], ctypes.c_char_p),
        "mf_get_launch_times": ([vp, vp, i64, ctypes.POINTER(i64)], ctypes.c_int),
        "mf_get_launch_timeline": ([vp, vp, vp, i64, ctypes.POINTER(i64)], ctypes.c_int),
        "mf_set_variant_model": ([vp, vp, i32, i32, i32], ctypes.c_int),
        "mf_get_variants": ([vp, vp], ctypes.c_int),
    }
    for name, (args, res) in sig.items():
        fn = getattr(L, name)
        fn.argtypes = args
        fn.restype = res
    return L


lib = _load()


class MfError(RuntimeError):
    def __init__(self, code: int, where: str):
        super().__init__(f"{where}: {lib.mf_strerror(code).decode()} ({code})")
        self.code = code


class MfNotSPD(MfError):
    def __init__(self, code: int, where: str, failed_col: int):
        super().__init__(code, where)
        self.failed_col = failed_col


def _ptr(x, dtype) -> int:
    """Raw pointer of a contiguous numpy array or torch tensor of ``dtype``."""
    if isinstance(x, np.ndarray):
        if x.dtype != dtype or not x.flags.c_contiguous:
            raise TypeError(f"expected contiguous {np.dtype(dtype)} array")
        return x.ctypes.data
    if hasattr(x, "data_ptr"):   # torch.Tensor (host or CUDA)
        import torch
        tdt = {np.float64: torch.float64, np.int32: torch.int32, np.int64: torch.int64}[np.dtype(dtype).type]
        if x.dtype != tdt or not x.is_contiguous():
            raise TypeError(f"expected contiguous {tdt} tensor")
        return x.data_ptr()
    raise TypeError(f"unsupported argument type {type(x)}")


class Solver:
    """mf_create / mf_analyze / mf_factor / mf_solve on one context."""

    def __init__(self, amalgamate: bool = True, small_front_max: int | None = None, panel_w: int | None = None,
                 device: int = -1, stream: int | None = None, host_only: bool = False,
                 nranks: int = 1, rank: int = 0, exchange=None, split_all: bool = False,
                 nbranch: int | None = None, fuse_ea: bool | None = None, lookahead: bool | None = None,
                 variant_model="auto", torch_alloc: bool = False, ozaki_slices: int = 0,
                 refine_iters: int | None = None, nrelax=None, zrelax=None):
        """variant_model: "auto" = the fitted kernel-variant selector packaged with the
        binding (selector.MODEL_PATH, Eqs. 3-5 fitted to B200 timings) when
        present, None = libmf's fixed front-order thresholds, or a theta array.
        Precedence: an explicit ``small_front_max`` selects the threshold policy
        ("auto" then resolves to None), since a variant model chooses each front's
        class by itself and would ignore the threshold (include/mf.h).
        torch_alloc: take every device buffer of the ctx from PyTorch's caching
        allocator (mf_options.dev_alloc / dev_free) instead of cudaMalloc.
        ozaki_slices: Schur updates on the int8 tensor cores (0 = FP64 DMMA, 8 =
        FP64-class Ozaki emulation, 3..7 = reduced precision + fp64 refinement in
        solve); refine_iters: max refinement steps (None = auto)."""
        if small_front_max is not None and isinstance(variant_model, str) and variant_model == "auto":
            variant_model = None
        o = Options()
        lib.mf_default_options(ctypes.byref(o))
        o.amalgamate = int(amalgamate)
        if nrelax is not None:   # relaxed-amalgamation thresholds (default {4,16,48})
            for i, v in enumerate(nrelax):
                o.nrelax[i] = int(v)
        if zrelax is not None:   # default {0.8, 0.1, 0.05}
            for i, v in enumerate(zrelax):
                o.zrelax[i] = float(v)
        if small_front_max is not None:
            o.small_front_max = small_front_max
        if panel_w is not None:
            o.panel_w = panel_w
        o.device = device
        o.host_only = int(host_only)
        o.nranks = nranks
        o.rank = rank
        o.split_all = int(split_all)
        if nbranch is not None:
            o.nbranch = nbranch
        if fuse_ea is not None:
            o.fuse_ea = int(fuse_ea)
        if lookahead is not None:
            o.lookahead = int(lookahead)
        o.stream = stream
        o.ozaki_slices = int(ozaki_slices)
        o.refine_iters = -1 if refine_iters is None else int(refine_iters)
        self._alloc_cbs = None
        if torch_alloc and not host_only:
            import torch
            dev = torch.cuda.current_device() if device < 0 else device

            def _alloc(nbytes, _user):
                try:
                    return torch.cuda.caching_allocator_alloc(int(nbytes), dev)
                except RuntimeError:
                    return None

            def _free(ptr, _user):
                torch.cuda.caching_allocator_delete(ptr)

            self._alloc_cbs = (DEV_ALLOC_FN(_alloc), DEV_FREE_FN(_free))
            o.dev_alloc = ctypes.cast(self._alloc_cbs[0], ctypes.c_void_p)
            o.dev_free = ctypes.cast(self._alloc_cbs[1], ctypes.c_void_p)
        h = ctypes.c_void_p()
        r = lib.mf_create(ctypes.byref(h), ctypes.byref(o))
        if r != MF_OK:
            raise MfError(r, "mf_create")
        self._h = h
        self.n = None
        self.nranks, self.rank = nranks, rank
        self._xcb = None
        self.variant_model = None
        if isinstance(variant_model, str) and variant_model == "auto":
            from . import selector as _sel   # (lazy: selector imports this module)
            th = _sel.load_model()
            if th is not None:
                self.set_variant_model(th)
                self.variant_model = _sel.MODEL_PATH
        elif variant_model is not None:
            self.set_variant_model(variant_model)
            self.variant_model = "caller theta"
        if exchange is not None:
            self.set_exchange(exchange)

    def set_exchange(self, fn):
        """fn(list of (op, peer, device_ptr, nbytes)) -> None; must complete the transfers."""
        def _cb(_user, ops, nops):
            try:
                fn([(ops[i].op, ops[i].peer, ops[i].ptr, ops[i].bytes) for i in range(nops)])
                return 0
            except Exception as e:  # noqa: BLE001 -- reported through the C return code
                import traceback
                traceback.print_exc()
                return 1
        self._xcb = EXCHANGE_FN(_cb)
        self._check(lib.mf_set_exchange(self._h, self._xcb, None), "mf_set_exchange")

    def mapping(self):
        inf = self.info()
        ns = inf["nsuper"]
        owner = np.empty(ns, dtype=np.int32)
        top = np.empty(ns, dtype=np.int8)
        load = np.empty(self.nranks, dtype=np.float64)
        tl = ctypes.c_double()
        self._check(lib.mf_get_mapping(self._h, owner.ctypes.data, top.ctypes.data, load.ctypes.data,
                                       ctypes.byref(tl)), "mf_get_mapping")
        self._top_kind = top
        return owner, top.astype(bool), load, tl.value

    def cooperative(self) -> np.ndarray:
        """Mask of the top supernodes factored cooperatively by all ranks."""
        self.mapping()
        return self._top_kind == 2

    def close(self):
        if getattr(self, "_h", None):
            lib.mf_destroy(self._h)
            self._h = None

    def __del__(self):
        self.close()

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()

    def _check(self, r, where):
        if r == MF_NOT_SPD:
            raise MfNotSPD(r, where, self.info()["failed_col"])
        if r != MF_OK:
            raise MfError(r, where)

    def analyze(self, n: int, colptr, rowind, perm=None):
        """perm: new -> old order, or None for the library's METIS nested dissection."""
        colptr = np.ascontiguousarray(colptr, dtype=np.int64)
        rowind = np.ascontiguousarray(rowind, dtype=np.int32)
        pp = None
        if perm is not None:
            perm = np.ascontiguousarray(perm, dtype=np.int32)
            pp = perm.ctypes.data
        self._check(lib.mf_analyze(self._h, int(n), colptr.ctypes.data, rowind.ctypes.data, pp), "mf_analyze")
        self.n = int(n)
        self._info = self.info()

    def factor(self, values):
        """values: float64 numpy array (host) or torch tensor (host or CUDA)."""
        self._check(lib.mf_factor(self._h, _ptr(values, np.float64)), "mf_factor")

    def solve(self, b, x=None):
        if x is None:
            x = np.empty(self.n, dtype=np.float64)
        self._check(lib.mf_solve(self._h, _ptr(b, np.float64), _ptr(x, np.float64)), "mf_solve")
        return x

    def info(self) -> dict:
        i = Info()
        self._check(lib.mf_get_info(self._h, ctypes.byref(i)), "mf_get_info")
        return i.as_dict()

    def perm(self) -> np.ndarray:
        p = np.empty(self.n, dtype=np.int32)
        self._check(lib.mf_get_perm(self._h, p.ctypes.data), "mf_get_perm")
        return p

    def etree(self):
        par = np.empty(self.n, dtype=np.int32)
        cc = np.empty(self.n, dtype=np.int64)
        self._check(lib.mf_get_etree(self._h, par.ctypes.data, cc.ctypes.data), "mf_get_etree")
        return par, cc

    def supernodes(self) -> dict:
        inf = self.info()
        ns, nf = inf["nsuper"], inf["nfund"]
        first = np.empty(ns + 1, dtype=np.int32)
        par = np.empty(ns, dtype=np.int32)
        rp = np.empty(ns + 1, dtype=np.int64)
        rows = np.empty(inf["rows_total"], dtype=np.int32)
        fund = np.empty(nf + 1, dtype=np.int32)
        self._check(lib.mf_get_supernodes(self._h, first.ctypes.data, par.ctypes.data, rp.ctypes.data,
                                          rows.ctypes.data, fund.ctypes.data), "mf_get_supernodes")
        return dict(sn_first=first, sn_parent=par, sn_rowptr=rp, sn_rows=rows, fund_first=fund)

    def panel(self, s: int, f: int, k: int) -> np.ndarray:
        """Panel of supernode s as an f x k array (column-major copy transposed to numpy order)."""
        out = np.empty(f * k, dtype=np.float64)
        self._check(lib.mf_export_panel(self._h, int(s), out.ctypes.data), "mf_export_panel")
        return out.reshape(k, f).T

    def program(self) -> list[dict]:
        cnt = ctypes.c_int64()
        self._check(lib.mf_get_program(self._h, None, 0, ctypes.byref(cnt)), "mf_get_program")
        arr = (LaunchInfo * max(cnt.value, 1))()
        self._check(lib.mf_get_program(self._h, arr, cnt.value, ctypes.byref(cnt)), "mf_get_program")
        return [dict(kind=a.kind, level=a.level, count=a.count, flops=a.flops, bytes=a.bytes, int8_ops=a.int8_ops,
                     stream=a.stream) for a in arr[:cnt.value]]

    def launch_times(self) -> np.ndarray:
        """CUDA-event ms of every launch of the last profiled factorization (program order)."""
        cnt = ctypes.c_int64()
        self._check(lib.mf_get_launch_times(self._h, None, 0, ctypes.byref(cnt)), "mf_get_launch_times")
        out = np.zeros(max(cnt.value, 1), dtype=np.float64)
        self._check(lib.mf_get_launch_times(self._h, out.ctypes.data, cnt.value, ctypes.byref(cnt)),
                    "mf_get_launch_times")
        return out[:cnt.value]

    def launch_timeline(self) -> tuple[np.ndarray, np.ndarray]:
        """(start_ms, end_ms) of every launch of the last factorization run with
        set_profiling(2): the concurrent graph's timeline (program order)."""
        cnt = ctypes.c_int64()
        self._check(lib.mf_get_launch_timeline(self._h, None, None, 0, ctypes.byref(cnt)), "mf_get_launch_timeline")
        t0 = np.zeros(max(cnt.value, 1), dtype=np.float64)
        t1 = np.zeros(max(cnt.value, 1), dtype=np.float64)
        self._check(lib.mf_get_launch_timeline(self._h, t0.ctypes.data, t1.ctypes.data, cnt.value,
                                               ctypes.byref(cnt)), "mf_get_launch_timeline")
        return t0[:cnt.value], t1[:cnt.value]

    def set_variant_model(self, theta=None, force: int = -1):
        """Kernel-variant selector (before analyze): theta (MF_VARIANT_FEATURES x MF_VARIANTS)
        or None for the default thresholds; force >= 0 forces a class where feasible."""
        if theta is None:
            self._check(lib.mf_set_variant_model(self._h, None, 0, 0, int(force)), "mf_set_variant_model")
            return
        th = np.ascontiguousarray(theta, dtype=np.float64)
        if th.shape != (MF_VARIANT_FEATURES, MF_VARIANTS):
            raise ValueError(f"theta must be {MF_VARIANT_FEATURES} x {MF_VARIANTS}")
        self._check(lib.mf_set_variant_model(self._h, th.ctypes.data, MF_VARIANT_FEATURES, MF_VARIANTS, int(force)),
                    "mf_set_variant_model")

    def variants(self) -> np.ndarray:
        out = np.empty(max(self._info["nsuper"], 1), dtype=np.int32)
        self._check(lib.mf_get_variants(self._h, out.ctypes.data), "mf_get_variants")
        return out[:self._info["nsuper"]]

    def set_profiling(self, enable: int = 1):
        """1 (True): eager per-launch timing; 2: timeline of the concurrent graph; 0: off."""
        self._check(lib.mf_set_profiling(self._h, int(enable)), "mf_set_profiling")

    def kernel_stats(self) -> list[dict]:
        arr = (KernelStat * MF_KERNEL_CLASSES)()
        cnt = ctypes.c_int32()
        self._check(lib.mf_get_kernel_stats(self._h, arr, ctypes.byref(cnt)), "mf_get_kernel_stats")
        return [dict(name=a.name.decode(), launches=a.launches, ms=a.ms, flops=a.flops, bytes=a.bytes)
                for a in arr[:cnt.value]]

    def diag(self) -> np.ndarray:
        out = np.empty(self.n, dtype=np.float64)
        self._check(lib.mf_export_diag(self._h, out.ctypes.data), "mf_export_diag")
        return out

    def export_panels(self, total_words: int) -> np.ndarray:
        """Every panel (supernode order, each f x k column-major) concatenated."""
        out = np.empty(total_words, dtype=np.float64)
        self._check(lib.mf_export_panels(self._h, out.ctypes.data), "mf_export_panels")
        return out

    def export_L(self, values: bool = True):
        """L in supernodal CSC (final-perm labels): (Lp int64[n+1], Li int32, Lx float64)."""
        Lp = np.empty(self.n + 1, dtype=np.int64)
        self._check(lib.mf_export_L(self._h, Lp.ctypes.data, None, None), "mf_export_L")
        Li = np.empty(int(Lp[-1]), dtype=np.int32)
        Lx = np.empty(int(Lp[-1]), dtype=np.float64) if values else None
        self._check(lib.mf_export_L(self._h, Lp.ctypes.data, Li.ctypes.data,
                                    None if Lx is None else Lx.ctypes.data), "mf_export_L")
        return Lp, Li, Lx

    def solve_nrhs(self, B, X=None):
        """X = A^{-1} B for an n x nrhs column-major (Fortran-order) B."""
        if isinstance(B, np.ndarray):
            B = np.asfortranarray(B, dtype=np.float64)
            if B.ndim == 1:
                B = B[:, None]
            if X is None:
                X = np.empty(B.shape, dtype=np.float64, order="F")
            nrhs, ldb, ldx = B.shape[1], B.shape[0], X.shape[0]
            bp, xp = B.ctypes.data, X.ctypes.data
        else:   # torch tensors: (nrhs, n) row-major = n x nrhs column-major
            nrhs, ldb = B.shape[0], B.shape[1]
            if X is None:
                X = B.new_empty(B.shape)
            ldx = X.shape[1]
            bp, xp = _ptr(B, np.float64), _ptr(X, np.float64)
        self._check(lib.mf_solve_nrhs(self._h, int(nrhs), bp, int(ldb), xp, int(ldx)), "mf_solve_nrhs")
        return X
