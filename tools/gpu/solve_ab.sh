# solve A/B: fused init threshold (MF_SOLVE_FUSE_INIT), targeted solve tests
timeout 900 python -m pytest tests -m gpu -q -x -k "solve or refine or nrhs or nanfill or multigpu or torchdist" > gpurun_out/solvetest.log 2>&1; tail -1 gpurun_out/solvetest.log
for e in 0 64 256 100000; do for c in c5 c3 c2; do MF_SOLVE_FUSE_INIT=$e timeout 300 python tools/solve_time.py $c | sed "s/^/fuse<=$e /"; done; done > gpurun_out/solve_ab.txt 2>&1
