set -x
python bench.py --steps 5 --warmup 3 > gpurun_out/bench.json 2> gpurun_out/bench.err; tail -3 gpurun_out/bench.err
cat gpurun_out/bench.json
ncu --metrics gpu__time_duration.sum --clock-control none --profile-from-start off --csv --log-file gpurun_out/launches.csv python tools/prof_factor.py c5 > gpurun_out/launches.log 2>&1; tail -2 gpurun_out/launches.log
ncu --set full --clock-control none --import-source on --profile-from-start off -k regex:k_update -s 300 -c 2 -o gpurun_out/prof_update python tools/prof_factor.py c5 > gpurun_out/ncu_full.log 2>&1; tail -3 gpurun_out/ncu_full.log
ls -la gpurun_out
