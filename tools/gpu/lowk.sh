timeout 1200 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -k "bulk or fused or grid" 2>&1 | tail -2
for c in c5 c3 c2; do for lk in 0 1; do MF_UPD_LOWK=$lk timeout 600 python tools/la_ab.py $c nbranch=4 2>&1 | sed "s/^/lowk=$lk /"; done; done
