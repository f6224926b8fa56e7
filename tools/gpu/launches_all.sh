set -x
for c in c5 c3 c4 c2; do
ncu --metrics gpu__time_duration.sum --clock-control none --profile-from-start off --csv --log-file gpurun_out/${c}_launches.csv python tools/prof_factor.py $c > gpurun_out/${c}_launches.log 2>&1
tail -1 gpurun_out/${c}_launches.log
done
for c in c1 c2 c3 c4; do python bench.py --config $c --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/bench_$c.json 2> gpurun_out/bench_$c.err; tail -1 gpurun_out/bench_$c.json | cut -c1-300; done
