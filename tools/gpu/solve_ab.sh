# solve A/B: forward chain shortcut (MF_SOLVE_M), targeted solve tests
timeout 900 python -m pytest tests -m gpu -q -x -k "solve or refine or nrhs or nanfill or multigpu or torchdist or manufactured" > gpurun_out/solvetest.log 2>&1; tail -1 gpurun_out/solvetest.log
for e in 0 1; do for c in c5 c3 c2; do MF_SOLVE_M=$e timeout 300 python tools/solve_time.py $c | sed "s/^/M=$e /"; done; done > gpurun_out/solve_ab.txt 2>&1
