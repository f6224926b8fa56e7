# look-ahead A/B: bit identity + lookahead=0,1 on c2-c5 + the dense calibration (MF_LA)
timeout 900 python -m pytest tests -m gpu -q -x -k "lookahead" > gpurun_out/la2_test.log 2>&1; tail -1 gpurun_out/la2_test.log
for c in c3 c5 c2 c4; do timeout 600 python tools/la_ab.py $c lookahead=0,1; done > gpurun_out/la2_ab.txt 2>&1
for la in 0 1; do MF_LA=$la timeout 600 python tools/dense_potrf.py 7014 14900 5418; done >> gpurun_out/la2_ab.txt 2>&1
