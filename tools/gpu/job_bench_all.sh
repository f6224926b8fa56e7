# bench lines of c2, c3, c4 (default steps) -> gpurun_out/bench_<c>.json
for c in c2 c3 c4; do timeout 900 python bench.py --config $c > gpurun_out/bench_$c.json 2> gpurun_out/bench_$c.err; tail -1 gpurun_out/bench_$c.json | cut -c1-200; done
