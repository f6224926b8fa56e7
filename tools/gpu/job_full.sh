# full GPU test suite, then the default bench line (c5)
timeout 2000 python -m pytest tests -m gpu -q -x > gpurun_out/gputest_full.log 2>&1; tail -2 gpurun_out/gputest_full.log
timeout 900 python bench.py > gpurun_out/bench_c5.json 2> gpurun_out/bench_c5.err; tail -c 3000 gpurun_out/bench_c5.json
