set -x
timeout 900 python -m pytest tests -m gpu -q -x -k "solve or refine or nrhs or nanfill or bulk or multigpu or torchdist" > gpurun_out/solvetest.log 2>&1; tail -3 gpurun_out/solvetest.log
for c in c5 c3 c2; do timeout 300 python tools/solve_time.py $c; done > gpurun_out/solve_time3.txt 2>&1
MF_SOLVE_SLOTS=1 timeout 300 python tools/solve_time.py c3 >> gpurun_out/solve_time3.txt 2>&1
cat gpurun_out/solve_time3.txt
