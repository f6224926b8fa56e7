set -x
ncu --metrics gpu__time_duration.sum --clock-control none --profile-from-start off --csv --log-file gpurun_out/c5_launches.csv python tools/prof_factor.py c5 > gpurun_out/c5_launches.log 2>&1
tail -2 gpurun_out/c5_launches.log
