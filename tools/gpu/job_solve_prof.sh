# per-launch device times of one warm c5 solve (ncu, cold caches, serialised)
ncu --metrics gpu__time_duration.sum --clock-control none --profile-from-start off --csv \
    --log-file gpurun_out/solve_launches_${1:-c5}.csv python tools/prof_solve.py ${1:-c5} > gpurun_out/solve_prof.log 2>&1
tail -2 gpurun_out/solve_prof.log
