./tools/ubench/panel_bench 14900 14900 4 | head -3
./tools/ubench/panel_bench 4000 4000 4 | head -1
./tools/ubench/panel_bench 4000 4000 4 | tail -1
./tools/ubench/panel_bench 1000 250 4 | tail -1
timeout 1200 python -m pytest tests/test_gpu_parity.py -x -q -m gpu 2>&1 | tail -2
for c in c5 c3 c4; do timeout 600 python tools/la_ab.py $c nbranch=4 2>&1; done
