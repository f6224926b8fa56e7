set -x
timeout 1500 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -k full_size 2>&1 | tail -5
for c in c1 c2 c3 c4; do python bench.py --config $c --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/bench_$c.json 2> gpurun_out/bench_$c.err; tail -2 gpurun_out/bench_$c.err; done
