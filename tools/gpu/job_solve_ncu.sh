# DRAM traffic and throughput of every solve launch of one warm c5 solve (ncu, cold caches)
ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none \
    --profile-from-start off --csv --log-file gpurun_out/solve_traffic_${1:-c5}.csv python tools/prof_solve.py ${1:-c5} > /dev/null 2>&1
tail -3 gpurun_out/solve_traffic_${1:-c5}.csv | cut -c1-150
