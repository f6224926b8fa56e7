# small-front threshold policy vs the learned selector on the latency-bound configs
for c in c2 c3; do timeout 600 python tools/time_factor.py $c; timeout 900 python tools/la_ab.py $c small_front_max=64,128,192,256; done > gpurun_out/sfm_ab.txt 2>&1
