"""Single-thread oracle seconds for configs c1-c3 ("Single-thread
time as well for configs 1-3") -> profiles/oracle_single_thread.json, which
bench.py's cpu_baseline reports.  Run on the GPU box's host:
    OMP_NUM_THREADS=1 python tools/oracle_single_thread.py"""
import json
import os
import platform
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
assert os.environ.get("OMP_NUM_THREADS") == "1", "run with OMP_NUM_THREADS=1"
import oracle  # noqa: E402
from workloads import grids as G  # noqa: E402

model = "unknown"
for ln in open("/proc/cpuinfo"):
    if ln.startswith("model name"):
        model = ln.split(":", 1)[1].strip()
        break
out = {"cpu_model": model, "threads": 1, "host": platform.node(), "configs": {}}
for name in ("c1", "c2", "c3"):
    c = G.CONFIGS[name]
    A, p = G.make_config(c["kind"], c["N"])
    sym = oracle.symbolic(A, p)
    t0 = time.perf_counter()
    n = sum(1 for _ in oracle.factor_stream(A, sym))
    dt = time.perf_counter() - t0
    out["configs"][name] = {"seconds": dt, "fronts": n, "flops_true": int(sym.flops),
                            "GFLOPs": sym.flops / dt / 1e9}
    print(name, out["configs"][name], flush=True)
dst = os.path.join(ROOT, "gpurun_out", "oracle_single_thread.json")
os.makedirs(os.path.dirname(dst), exist_ok=True)
json.dump(out, open(dst, "w"), indent=1)
