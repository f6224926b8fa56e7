set -x
for c in c5 c3; do timeout 600 python tools/level_breakdown.py $c 1 > gpurun_out/levels_${c}.txt 2>&1; tail -3 gpurun_out/levels_${c}.txt; done
ncu --metrics gpu__time_duration.sum --clock-control none --profile-from-start off --csv --log-file gpurun_out/c5_launches.csv python tools/prof_factor.py c5 > gpurun_out/c5_launches.log 2>&1
tail -2 gpurun_out/c5_launches.log
