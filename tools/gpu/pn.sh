./tools/ubench/panel_bench 14900 14900 4 | head -1
./tools/ubench/panel_bench 4000 4000 4 | head -1
timeout 1200 python -m pytest tests/test_gpu_parity.py -x -q -m gpu 2>&1 | tail -2
for c in c5 c3 c4 c2; do timeout 600 python bench.py --config $c --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/bench_$c.json 2> gpurun_out/bench_$c.err; tail -1 gpurun_out/bench_$c.err; python -c "import json;d=json.load(open('gpurun_out/bench_$c.json'));print('$c', round(d['ms_per_step'],3), 'ms', round(d['value']), 'e2e', round(d['e2e']['value']), [(k['name'], round(k['ms']/d['steps'],2)) for k in d['kernels'] if k['ms']>0])"; done
