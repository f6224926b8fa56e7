set -x
timeout 900 python -m pytest tests -x -q -m gpu > gpurun_out/pytest_gpu.log 2>&1; tail -15 gpurun_out/pytest_gpu.log
timeout 600 python tools/dense_potrf.py > gpurun_out/dense_potrf.log 2>&1; cat gpurun_out/dense_potrf.log
for c in c5 c3 c2; do timeout 600 python bench.py --config $c --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/bench_$c.json 2> gpurun_out/bench_$c.err; tail -2 gpurun_out/bench_$c.err; cut -c1-400 gpurun_out/bench_$c.json; done
