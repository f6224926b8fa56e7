timeout 300 ./tools/ubench/update_variants 8192 4096 2>&1 | head -3
./tools/ubench/update_trap 16 3000 256 256 10 | tail -1
timeout 1200 python -m pytest tests/test_gpu_parity.py -x -q -m gpu 2>&1 | tail -1
for c in c5 c3 c4 c2; do timeout 600 python tools/la_ab.py $c nbranch=4 2>&1; done
