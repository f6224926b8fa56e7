set -x
ncu --metrics gpu__time_duration.sum --clock-control none --profile-from-start off --csv --log-file gpurun_out/dense5418_launches.csv python tools/dense_potrf.py --prof 5418 > gpurun_out/dense_prof.log 2>&1; tail -2 gpurun_out/dense_prof.log
ncu --set full --clock-control none --import-source on --profile-from-start off -k regex:k_panel -s 30 -c 1 -o gpurun_out/prof_panel python tools/dense_potrf.py --prof 5418 > gpurun_out/ncu_panel.log 2>&1; tail -1 gpurun_out/ncu_panel.log
