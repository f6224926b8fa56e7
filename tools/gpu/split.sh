timeout 1200 python -m pytest tests/test_gpu_parity.py -x -q -m gpu 2>&1 | tail -1
for c in c5 c3 c4 c2; do for a in 0 1; do MF_SPLIT_ALIGN=$a timeout 600 python tools/la_ab.py $c nbranch=4 2>&1 | sed "s/^/align=$a /"; done; done
