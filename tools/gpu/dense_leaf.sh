set -x
timeout 600 python tools/dense_potrf.py > gpurun_out/dense_potrf.log 2>&1; cat gpurun_out/dense_potrf.log
ncu --set full --clock-control none --import-source on --profile-from-start off -k regex:k_leaf -s 380 -c 1 -o gpurun_out/prof_leaf python tools/prof_factor.py c5 > gpurun_out/ncu_leaf.log 2>&1; tail -1 gpurun_out/ncu_leaf.log
