# solve: targeted solve tests + device solve times of c5 / c3 / c2 / c4 (A/B driver)
timeout 900 python -m pytest tests -m gpu -q -x -k "solve or refine or nrhs or nanfill or multigpu or torchdist or manufactured" > gpurun_out/solvetest.log 2>&1; tail -1 gpurun_out/solvetest.log
for c in c5 c3 c2 c4; do timeout 300 python tools/solve_time.py $c; done > gpurun_out/solve_ab.txt 2>&1
