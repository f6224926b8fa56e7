"""Timeline of one factorization as its CUDA graph runs (mf_set_profiling(2):
timing events captured before / after every launch; subtree branches and streams
concurrent) -- where the wall time of a config goes, launch by launch.

    python tools/timeline.py c2 [--csv out.csv]          (GPU)

Prints the makespan, each stream's busy span, and the launches of the main
stream (the top of the tree after the branches join) with their start / end;
with --csv, every launch (index, stream, level, kind, tasks, start, end)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_ipps_georgesgsc11_b200 as mf  # noqa: E402
from workloads import grids as G  # noqa: E402

NAMES = {0: "small", 1: "assemble", 2: "potrf", 3: "trsm", 4: "update", 5: "leaf", 6: "panel"}


def main():
    cfg = sys.argv[1] if len(sys.argv) > 1 else "c2"
    out_csv = sys.argv[sys.argv.index("--csv") + 1] if "--csv" in sys.argv else None
    c = G.CONFIGS[cfg]
    A, p = G.make_config(c["kind"], c["N"])
    S = mf.Solver()
    S.analyze(A.n, A.colptr, A.rowind, p)
    v = torch.from_numpy(A.values).cuda()
    for _ in range(3):
        S.factor(v)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    S.factor(v)
    e1.record()
    torch.cuda.synchronize()
    plain = e0.elapsed_time(e1)
    S.set_profiling(2)
    S.factor(v)   # captures the timeline graph
    S.factor(v)
    torch.cuda.synchronize()
    t0, t1 = S.launch_timeline()
    prog = S.program()
    span = float(t1.max())
    print(f"{cfg}: plain graph {plain:.3f} ms; timeline graph {span:.3f} ms (events add a little); "
          f"{len(prog)} launches")
    streams = sorted({L["stream"] for L in prog})
    for st in streams:
        idx = [i for i, L in enumerate(prog) if L["stream"] == st]
        busy = float(np.sum(t1[idx] - t0[idx]))
        print(f"  stream {st:2d}: {len(idx):4d} launches, span {t0[idx].min():8.3f} .. {t1[idx].max():8.3f} ms, "
              f"sum of launch times {busy:8.3f} ms")
    byk = {}
    for i, L in enumerate(prog):
        k = (L["stream"] < 0, NAMES.get(L["kind"], str(L["kind"])))
        byk[k] = byk.get(k, 0.0) + float(t1[i] - t0[i])
    print("  launch time by class (main stream / branches):",
          {f"{'main' if m else 'branch'}:{n}": round(t, 3) for (m, n), t in sorted(byk.items())})
    main_idx = [i for i, L in enumerate(prog) if L["stream"] < 0]
    if main_idx:
        print("  main stream (after the branches join):")
        for i in main_idx:
            L = prog[i]
            print(f"    #{i:4d} L{L['level']:2d} {NAMES.get(L['kind'], L['kind']):9s} tasks {L['count']:6d} "
                  f"{t0[i]:8.3f} -> {t1[i]:8.3f} ms ({(t1[i] - t0[i]) * 1e3:7.1f} us)")
    if out_csv:
        with open(out_csv, "w") as fh:
            fh.write("index,stream,level,kind,tasks,flops,start_ms,end_ms\n")
            for i, L in enumerate(prog):
                fh.write(f"{i},{L['stream']},{L['level']},{NAMES.get(L['kind'], L['kind'])},{L['count']},"
                         f"{L['flops']:.6g},{t0[i]:.6f},{t1[i]:.6f}\n")
    S.close()


if __name__ == "__main__":
    main()
