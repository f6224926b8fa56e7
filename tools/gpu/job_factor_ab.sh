# targeted factor tests (bit-identity of the fused extend-add, manufactured, parity) + bench lines
timeout 1200 python -m pytest tests -m gpu -q -x -k "fused or manufactured or bulk or grid or parity or variant" > gpurun_out/factortest.log 2>&1; tail -1 gpurun_out/factortest.log
for c in ${@:-c2 c3 c4 c5}; do timeout 600 python bench.py --config $c --steps 10 --warmup 3 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$c', round(d['ms_per_step'],3), 'ms', round(d['value']), d['unit'])"; done
