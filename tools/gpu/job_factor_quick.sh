# targeted factor tests + c2/c3 bench lines (fast A/B of factor-kernel changes)
timeout 900 python -m pytest tests -m gpu -q -x -k "tiny or small or manufactured or variant or parity or nanfill" > gpurun_out/factortest.log 2>&1; tail -2 gpurun_out/factortest.log
for c in ${@:-c2 c3}; do timeout 600 python bench.py --config $c --steps 10 --warmup 3 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$c', round(d['ms_per_step'],3), 'ms', d['value'], d['unit'])"; done
