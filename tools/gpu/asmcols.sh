timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -k "grid or fused or full_size" 2>&1 | tail -1
for c in c5 c4 c3 c2; do timeout 600 python tools/la_ab.py $c nbranch=4 2>&1; done
