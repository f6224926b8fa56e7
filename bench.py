#!/usr/bin/env python
"""bench.py -- fp64 multifrontal sparse Cholesky factorization throughput on B200.

Metric (BASELINE.json): "fp64 factorization GFLOP/s and seconds at 1/2/4/8 B200
(% of FP64 TC peak)".  A step = one mf_factor (the whole hot path: every front's
assembly/extend-add, potrf, trsm and Schur update) of the N=1 workload, the
north-star target "3D 27-point stencil 100^3 (n=1M), nested dissection"
(BASELINE.json configs[4], `--config c5`, the default).  GFLOP/s counts the
algorithmic flops of the TRUE factor, sum_j cc_j^2.

    python bench.py [--gpus N --steps K --warmup W] [--config c5] [--impl reference]

Multi-GPU (torchrun, one rank per GPU): the SAME matrix is factored by all
ranks together -- elimination subtrees mapped subtree-to-GPU, the supernodes
above them replicated on every rank (the large ones factored cooperatively,
pivot-column blocks broadcast over NCCL by their owner) -- so this is strong
scaling ("scaling": "strong"); DESIGN.md "Multi-GPU" states the modelled bound.
"""
from __future__ import annotations

import argparse
import json
import os
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

from workloads import grids as G  # noqa: E402

PEAK_NOMINAL_FP64 = 37.2e12   # 148 SM x 64 FP64 FMA/clk x 2 x 1.965 GHz


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--config", default="c5", choices=sorted(G.CONFIGS))
    ap.add_argument("--impl", default="mf", choices=["mf", "reference"])
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-modes", action="store_true", help="skip the Ozaki int8 Schur-update mode lines")
    ap.add_argument("--cpu-sample-gflop", type=float, default=170.0,
                    help="--impl reference: true GFLOP of the oracle sample per step (one whole subtree)")
    ap.add_argument("--cpu-baseline-gflop", type=float, default=1500.0,
                    help="cpu_baseline of the product arm: true GFLOP of its one-off oracle sample (~10-30 s)")
    ap.add_argument("--small-front-max", type=int, default=None)
    ap.add_argument("--panel-w", type=int, default=None)
    ap.add_argument("--nbranch", type=int, default=None, help="concurrent subtree branches (single GPU)")
    return ap.parse_args()


# ------------------------------------------------------------------ clocks
class ClockSampler:
    """nvidia-smi sampling DURING the timed region (B200_PROFILING.md clocks line)."""
    FIELDS = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
              "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
              "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, gpu: int):
        self.gpu = gpu
        self.proc = None
        self.lines: list[str] = []

    def start(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", "-i", str(self.gpu), f"--query-gpu={self.FIELDS}",
                                          "--format=csv,noheader,nounits", "-lms", "100"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except OSError:
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    def stop(self) -> dict:
        if self.proc is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        time.sleep(0.15)
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except subprocess.TimeoutExpired:
            self.proc.kill()
        sm, smax, reasons, power = [], [], set(), []
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in self.lines:
            parts = [x.strip() for x in ln.split(",")]
            if len(parts) < 9:
                continue
            try:
                sm.append(float(parts[1]))
                smax.append(float(parts[2]))
                power.append(float(parts[3]))
            except ValueError:
                continue
            for nm, v in zip(names, parts[5:9]):
                if v.lower() == "active":
                    reasons.add(nm)
        return {"sm_mhz": float(np.median(sm)) if sm else None, "sm_max_mhz": max(smax) if smax else None,
                "reasons": sorted(reasons), "samples": len(sm), "power_w_max": max(power) if power else None}


# ------------------------------------------------------------------ helpers
def dist_env():
    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return rank, world, local


def measured_dgemm_peak(torch) -> float:
    """cuBLAS DGEMM 8192^3 burst on this GPU (the fp64 roofline denominator;
    MEASURED_PEAKS.json has no fp64 figure)."""
    n = 8192
    a = torch.randn(n, n, dtype=torch.float64, device="cuda")
    b = torch.randn(n, n, dtype=torch.float64, device="cuda")
    for _ in range(2):
        a @ b
    torch.cuda.synchronize()
    best = 1e9
    e0 = torch.cuda.Event(enable_timing=True)
    e1 = torch.cuda.Event(enable_timing=True)
    for _ in range(5):
        e0.record()
        a @ b
        e1.record()
        torch.cuda.synchronize()
        best = min(best, e0.elapsed_time(e1))
    del a, b
    torch.cuda.empty_cache()
    return 2.0 * n ** 3 / (best * 1e-3)


def oracle_sample(A, perm, target_gflop: float):
    """The bounded CPU sample: one whole elimination subtree of the workload
    (closed under descendants, so the oracle factors it exactly as in the full run)."""
    import oracle
    sym = oracle.symbolic(A, perm)
    ch = sym.children()
    cc = sym.cc.astype(np.float64)
    first = sym.sn_first
    own = np.array([np.sum(cc[first[s]:first[s + 1]] ** 2) for s in range(sym.nsuper)])
    sub = own.copy()
    for s in range(sym.nsuper):
        for q in ch[s]:
            sub[s] += sub[q]
    r = int(np.argmin(np.abs(sub - target_gflop * 1e9)))
    subset, stack = [], [r]
    while stack:
        v = stack.pop()
        subset.append(v)
        stack.extend(ch[v])
    return sym, sorted(subset), float(sub[r]), r


def run_oracle_steps(A, sym, subset, steps: int):
    import oracle
    times = []
    for _ in range(steps):
        t0 = time.perf_counter()
        oracle.factor(A, sym, subset=subset)
        times.append(time.perf_counter() - t0)
    return times


def cpu_cores() -> int:
    """Threads the oracle's OpenMP loops use (oracle/numeric.c: the default team,
    OMP_NUM_THREADS or every host core)."""
    env = os.environ.get("OMP_NUM_THREADS")
    return int(env) if env and env.isdigit() else (len(os.sched_getaffinity(0)) or 1)


def cpu_model() -> str:
    try:
        for ln in open("/proc/cpuinfo"):
            if ln.startswith("model name"):
                return ln.split(":", 1)[1].strip()
    except OSError:
        pass
    return "unknown"


def single_thread_reference() -> dict | None:
    """Single-thread oracle seconds for c1-c3 (tools/oracle_single_thread.py on
    the GPU box's host, committed under profiles/): a fixed measurement, not
    re-run by every bench."""
    try:
        return json.load(open(os.path.join(ROOT, "profiles", "oracle_single_thread.json")))
    except (OSError, ValueError):
        return None


def traffic_for(cfg: str, kernel: str, launches_per_step: int):
    """ncu DRAM bytes per launch of `kernel` for THIS program (profiles/ncu_traffic_<cfg>.json,
    tools/gpu/profile.sh) -- refused when the capture's launch count differs from
    the benched program's."""
    path = os.path.join(ROOT, "profiles", f"ncu_traffic_{cfg}.json")
    try:
        prof = json.load(open(path))
    except (OSError, ValueError):
        return None, f"no {os.path.basename(path)}"
    k = prof.get("kernels", {}).get(kernel)
    if not k:
        return None, f"{kernel} not in {os.path.basename(path)}"
    if k.get("launches") != launches_per_step:
        return None, (f"{os.path.basename(path)} has {k.get('launches')} {kernel} launches, "
                      f"the benched program {launches_per_step}: stale capture refused")
    return k["dram_bytes_per_launch"], os.path.basename(path)


# ------------------------------------------------------------------ reference arm
def run_reference(args):
    rank, world, _ = dist_env()
    if rank != 0:
        return 0
    c = G.CONFIGS[args.config]
    A, perm = G.make_config(c["kind"], c["N"])
    sym, subset, gflop, root = oracle_sample(A, perm, args.cpu_sample_gflop)
    run_oracle_steps(A, sym, subset, args.warmup)
    times = run_oracle_steps(A, sym, subset, args.steps)
    t = float(np.mean(times))
    value = gflop / t / 1e9
    sample = (f"oracle.factor of the whole elimination subtree rooted at supernode {root} "
              f"({len(subset)} fronts, {gflop:.3e} true flops) of {args.config}, incl. B assembly")
    line = {
        "impl": "reference", "metric": "fp64 factorization GFLOP/s", "value": value, "unit": "GFLOP/s",
        "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup, "ms_per_step": t * 1e3,
        "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
        "config": {"workload": c["desc"] + f" [{args.config}], CPU oracle sample", "n": A.n},
        "cpu_baseline": {"value": value, "unit": "GFLOP/s", "cores": cpu_cores(), "kind": "oracle", "sample": sample,
                         "cpu_model": cpu_model()},
        "e2e": {"value": value, "unit": "GFLOP/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
        "gpu_launches": 0,
    }
    print(json.dumps(line), flush=True)
    return 0


# ------------------------------------------------------------------ Schur-update modes (NEXT-3)
def int8_peak_tops() -> tuple[float, str]:
    """Dense int8 tensor peak: MEASURED_PEAKS.json bf16 burst x 2 (the guide's
    nominal int8 : bf16 ratio, 4.5 : 2.25 POPS), else the nominal 4.5 POPS."""
    try:
        bf16 = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))["bf16_tflops"]
        return 2.0 * bf16, "MEASURED_PEAKS.json bf16_tflops (burst) x 2 (nominal int8/bf16 ratio)"
    except (OSError, ValueError, KeyError):
        return 4500.0, "nominal 4.5 POPS dense int8 (no MEASURED_PEAKS.json)"


def bench_mode(torch, mf, A, perm, vals_d, stream, slices: int, steps: int, warmup: int, b=None):
    """One Schur-update mode (mf_options.ozaki_slices) on the same workload: device
    time per factorization, the int8 tensor-core launches' roofline, and -- when
    b is given -- the mixed-precision solve with fp64 refinement."""
    S = mf.Solver(stream=stream.cuda_stream, ozaki_slices=slices)
    S.analyze(A.n, A.colptr, A.rowind, perm)
    for _ in range(max(warmup, 3)):
        S.factor(vals_d)
    torch.cuda.synchronize()
    e0 = torch.cuda.Event(enable_timing=True)
    e1 = torch.cuda.Event(enable_timing=True)
    e0.record(stream)
    for _ in range(steps):
        S.factor(vals_d)
    e1.record(stream)
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / steps
    info = S.info()
    S.set_profiling(True)
    S.factor(vals_d)
    prog, times = S.program(), S.launch_times()
    S.set_profiling(False)
    oz = [i for i, L in enumerate(prog) if L["int8_ops"] > 0]
    t_oz = float(sum(times[i] for i in oz))
    ops = float(sum(prog[i]["int8_ops"] for i in oz))
    peak, src = int8_peak_tops()
    out = {"ozaki_slices": slices, "ms_per_step": ms, "value": info["flops_true"] / (ms * 1e-3) / 1e9,
           "unit": "GFLOP/s (fp64-equivalent, true-L flops)", "int8_launches": len(oz),
           "int8_launch_ms": t_oz, "int8_share_of_step": t_oz / (S.info()["t_factor"] * 1e3),
           "roofline_int8": {"bound": "tensor", "achieved": ops / (t_oz * 1e-3) / 1e12 if t_oz else None,
                             "peak": peak, "unit": "TOPS (int8 MMA ops executed)",
                             "frac": (ops / (t_oz * 1e-3) / 1e12) / peak if t_oz else None, "peak_source": src,
                             "fp64_equiv_TFLOPs": float(sum(prog[i]["flops"] for i in oz)) / (t_oz * 1e-3) / 1e12
                             if t_oz else None}}
    if b is not None:
        x = S.solve(b)
        inf = S.info()
        out["solve"] = {"refine_steps": inf["refine_steps"], "backward_error": inf["solve_berr"],
                        "solve_ms": inf["t_solve"] * 1e3,
                        "e2e_ms": ms + inf["t_solve"] * 1e3,
                        "what": "factor (reduced-precision Schur updates) + solve with fp64 iterative refinement; "
                                "backward error ||b-Ax||/(||A|| ||x|| + ||b||) (inf norms) computed on the GPU"}
        del x
    S.close()
    torch.cuda.empty_cache()
    return out


# ------------------------------------------------------------------ product arm
def main():
    args = parse()
    if args.impl == "reference":
        return run_reference(args)
    rank, world, local = dist_env()
    import torch
    if world > 1:
        import torch.distributed as dist
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    torch.cuda.set_device(local)
    import paper_conf_ipps_georgesgsc11_b200 as mf

    c = G.CONFIGS[args.config]
    A, perm = G.make_config(c["kind"], c["N"])
    stream = torch.cuda.Stream()
    exchange = None
    if world > 1:
        from paper_conf_ipps_georgesgsc11_b200.exchange import TorchDistExchange
        exchange = TorchDistExchange()
    S = mf.Solver(device=local, stream=stream.cuda_stream, small_front_max=args.small_front_max,
                  panel_w=args.panel_w, nranks=world, rank=rank, exchange=exchange, nbranch=args.nbranch)
    S.analyze(A.n, A.colptr, A.rowind, perm)
    info = S.info()
    flops = float(info["flops_true"])
    mapping = None
    if world > 1:
        _, top, load, top_load = S.mapping()
        coop = S.cooperative()
        sn = S.supernodes()
        k = np.diff(sn["sn_first"]).astype(float)
        m = np.diff(sn["sn_rowptr"]).astype(float) - k
        fl = k * m * m + m * k * (k + 1) + k * (k + 1) * (2 * k + 1) / 6
        tot = float(load.sum() + top_load)
        # flop bound (no exchange cost): subtrees in parallel, then the shared top
        # fronts split over the ranks and the replicated ones redundantly
        top_time = float(fl[coop].sum()) / world + float(fl[top & ~coop].sum())
        mapping = {"top_supernodes": int(top.sum()), "cooperative_top_supernodes": int(coop.sum()),
                   "top_flop_share": top_load / tot, "max_rank_subtree_share": float(load.max()) / tot,
                   "flop_bound_speedup": tot / (float(load.max()) + top_time)}
    vals_d = torch.from_numpy(A.values).cuda()
    torch.cuda.synchronize()

    def barrier():
        if world > 1:
            torch.distributed.barrier()

    for _ in range(max(args.warmup, 3)):
        S.factor(vals_d)
    barrier()
    torch.cuda.synchronize()
    sampler = ClockSampler(local)
    sampler.start()
    time.sleep(0.3)
    e0 = torch.cuda.Event(enable_timing=True)
    e1 = torch.cuda.Event(enable_timing=True)
    barrier()
    torch.cuda.synchronize()
    e0.record(stream)
    for _ in range(args.steps):
        S.factor(vals_d)
    e1.record(stream)
    torch.cuda.synchronize()
    barrier()
    clocks = sampler.stop()
    ms = e0.elapsed_time(e1) / args.steps
    # per-kernel CUDA-event timing: the same steps again with one event pair per
    # launch on the ctx stream (eager launches instead of the CUDA graph)
    S.set_profiling(True)
    for _ in range(args.steps):
        S.factor(vals_d)
    torch.cuda.synchronize()
    stats = S.kernel_stats()
    prof_ms = S.info()["t_factor"] * 1e3
    S.set_profiling(False)
    info = S.info()
    if world > 1:
        t = torch.tensor([ms], device="cuda", dtype=torch.float64)
        torch.distributed.all_reduce(t, op=torch.distributed.ReduceOp.MAX)
        ms = float(t.item())
    value = flops / (ms * 1e-3) / 1e9   # one matrix factored by all ranks together

    # ---- end to end through the C ABI with HOST buffers (pinned), factor + solve
    vals_h = torch.from_numpy(A.values).pin_memory()
    b_h = torch.from_numpy(G.rhs(A.n, 0)).pin_memory()
    x_h = torch.empty(A.n, dtype=torch.float64).pin_memory()
    S.factor(vals_h)
    S.solve(b_h, x_h)
    barrier()
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    for _ in range(args.steps):
        S.factor(vals_h)
        S.solve(b_h, x_h)
    t_e2e = (time.perf_counter() - t0) / args.steps
    if world > 1:
        t = torch.tensor([t_e2e], device="cuda", dtype=torch.float64)
        torch.distributed.all_reduce(t, op=torch.distributed.ReduceOp.MAX)
        t_e2e = float(t.item())
    t_solve = S.info()["t_solve"]
    # ---- the solve on the device (NEXT-2): one right-hand side, and 8 through
    # mf_solve_nrhs (concurrent solve pipelines), against reading the stored L twice
    solve = None
    if world == 1:
        bd = torch.from_numpy(G.rhs(A.n, 0)).cuda()
        xd = torch.empty_like(bd)
        S.solve(bd, xd)
        ts = []
        for _ in range(3):
            S.solve(bd, xd)
            ts.append(S.info()["t_solve"] * 1e3)
        B8 = torch.from_numpy(np.random.default_rng(1).uniform(-1, 1, (8, A.n))).cuda()
        S.solve_nrhs(B8)
        S.solve_nrhs(B8)
        t8 = S.info()["t_solve"] * 1e3
        hbm = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))["hbm_gbs"] \
            if os.path.exists(os.path.join(ROOT, "MEASURED_PEAKS.json")) else 6650.0
        bound = 2.0 * info["panel_words"] * 8 / (hbm * 1e9) * 1e3
        solve = {"ms_1rhs": float(np.median(ts)), "ms_per_rhs_nrhs8": t8 / 8, "hbm_bound_ms": bound,
                 "frac_1rhs": bound / float(np.median(ts)), "frac_nrhs8": bound / (t8 / 8),
                 "what": "device b/x; bound = 2 x stored L bytes / measured HBM GB/s"}
        del bd, xd, B8

    # ---- roofline of the dominant kernel (by event time inside the timed region)
    dom = max(stats, key=lambda s: s["ms"])
    peak_meas = measured_dgemm_peak(torch)
    traffic, traffic_src = traffic_for(args.config, dom["name"], dom["launches"] // max(args.steps, 1))
    if dom["name"] == "dmma_schur_update":
        achieved = dom["flops"] / (dom["ms"] * 1e-3) / 1e12
        roof = {"kernel": dom["name"], "bound": "tensor", "achieved": achieved, "peak": peak_meas / 1e12,
                "unit": "TFLOP/s", "frac": achieved / (peak_meas / 1e12), "traffic": traffic,
                "traffic_source": traffic_src,
                "peak_source": "cuBLAS DGEMM 8192^3 burst measured in this run (fp64 DMMA path)",
                "frac_of_nominal_37.2": achieved / (PEAK_NOMINAL_FP64 / 1e12),
                "launches": dom["launches"] // max(args.steps, 1), "share_of_step": dom["ms"] / (prof_ms * args.steps),
                "timing": "CUDA events around every launch on the ctx stream, profiled replay of the timed steps"}
    else:
        hbm = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))["hbm_gbs"] \
            if os.path.exists(os.path.join(ROOT, "MEASURED_PEAKS.json")) else 6650.0
        achieved = dom["bytes"] / (dom["ms"] * 1e-3) / 1e9
        roof = {"kernel": dom["name"], "bound": "hbm", "achieved": achieved, "peak": hbm, "unit": "GB/s",
                "frac": achieved / hbm, "traffic": traffic, "traffic_source": traffic_src,
                "launches": dom["launches"] // max(args.steps, 1), "share_of_step": dom["ms"] / (prof_ms * args.steps)}

    line = {
        "metric": "fp64 factorization GFLOP/s", "value": value, "unit": "GFLOP/s", "n_gpus": world,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms, "seconds_per_factorization": ms * 1e-3,
        "higher_is_better": True, "scaling": "strong" if world > 1 else "weak", "vs_baseline": None,
        "dtype": "f64", "data": "synthetic",
        "pct_of_fp64_peak": {"nominal_37.2TF": value / (world * PEAK_NOMINAL_FP64 / 1e9),
                             "measured_dgemm": value / (world * peak_meas / 1e9)},
        "config": {"workload": c["desc"] + f" [{args.config}]", "n": A.n, "nnz_lower": A.nnz,
                   "flops_true": flops, "flops_exec": float(info["flops_exec"]), "nsuper": info["nsuper"],
                   "max_front": info["max_front"],
                   "parallelism": (f"subtree-to-GPU x{world}, top fronts replicated and factored cooperatively "
                                   "(NCCL broadcasts)"
                                   if world > 1 else f"1 GPU, {info['nbranch']} concurrent subtree branches"),
                   "variant_selector": ("learned (PAPER Eqs. 3-5, " + os.path.basename(S.variant_model) + ")"
                                        if S.variant_model else "front-order thresholds"),
                   "l2": "no flush: working set (L = %.1f GB) >> 126 MB L2" % (info["panel_words"] * 8 / 1e9)},
        "clocks": clocks,
        "mapping": mapping,
        "e2e": {"value": flops / t_e2e / 1e9, "unit": "GFLOP/s",
                "what": "mf_factor(host pinned values) + mf_solve(host b -> host x), host wall",
                "seconds": t_e2e, "solve_seconds": t_solve,
                "h2d_bytes_per_step": int(A.nnz * 8 + A.n * 8), "d2h_bytes_per_step": int(A.n * 8 + 4)},
        "gpu_launches": int(info["launches_factor"]) * args.steps,
        "solve": solve,
        "roofline": roof,
        "kernels": [{k: (round(v, 4) if isinstance(v, float) else v) for k, v in s.items()} for s in stats],
        "profiled_ms_per_step": prof_ms,
    }
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        import oracle
        sym, subset, gflop, root = oracle_sample(A, perm, args.cpu_baseline_gflop)
        t0 = time.perf_counter()
        panels = oracle.factor(A, sym, subset=subset)
        t_or = time.perf_counter() - t0
        line["cpu_baseline"] = {
            "value": gflop / t_or / 1e9, "unit": "GFLOP/s", "cores": cpu_cores(), "kind": "oracle",
            "cpu_model": cpu_model(),
            "sample": (f"oracle.factor (plain C + OpenMP, no BLAS) of the whole elimination subtree rooted at "
                       f"supernode {root} ({len(subset)} fronts, {gflop:.3e} true flops) of {args.config}, "
                       "incl. B assembly"),
            "seconds": t_or, "single_thread_c1_c3": single_thread_reference()}
        # parity of the benched factor on that sample: every panel of the subtree
        sys.path.insert(0, os.path.join(ROOT, "tests"))
        from tests._parity import ParityStats
        st = ParityStats()
        for sn, Po in panels.items():
            st.add(sn, S.panel(sn, *Po.shape), Po, m_matrix=c["kind"] != "elast")
        rep = st.report()
        line["parity"] = dict(rep, what=("GPU panels of the benched factorization vs the oracle's on the "
                                          "cpu_baseline sample subtree; reading C11 (tests/_parity.py)"),
                              ok=rep["floored_max"] <= 1e-10)
        del panels
    if world == 1 and not args.no_modes:
        # NEXT-3 modes on the same workload (the fp64 DMMA line above is the headline)
        S.close()
        torch.cuda.empty_cache()
        modes = {}
        for key, sl, rhs in (("ozaki8_fp64_emulated", 8, None), ("ozaki4_mixed_refined", 4, G.rhs(A.n, 0))):
            try:   # an optional mode must never cost the headline line
                modes[key] = bench_mode(torch, mf, A, perm, vals_d, stream, sl, args.steps, args.warmup, b=rhs)
            except Exception as e:  # noqa: BLE001
                modes[key] = {"error": f"{type(e).__name__}: {e}"}
                torch.cuda.empty_cache()
        line["schur_modes"] = modes
    if rank == 0:
        print(json.dumps(line), flush=True)
    if world > 1:
        torch.distributed.destroy_process_group()
    return 0


if __name__ == "__main__":
    sys.exit(main())
