# A/B of the solve's small-front threshold (MF_SOLVE_SMALL, MF_SOLVE_SMALL_K)
for v in 16 32 64 256; do for c in c5 c3 c2; do echo "small 256 k<=$v: $(MF_SOLVE_SMALL_K=$v timeout 300 python tools/solve_time.py $c)"; done; done > gpurun_out/solve_small.txt 2>&1
cat gpurun_out/solve_small.txt
