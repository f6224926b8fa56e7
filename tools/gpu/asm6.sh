timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -k "grid or fused or full_size" 2>&1 | tail -1
for c in c5 c3 c4 c2; do timeout 600 python tools/la_ab.py $c nbranch=4 2>&1; done
NB=1 timeout 600 python tools/level_breakdown.py c5 1 2>&1 | grep -o "L1[2-8] assemble:[^|]*"
