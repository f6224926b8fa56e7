#!/bin/bash
# Evidence for one config (run under gpurun; copy the outputs into profiles/):
#   tools/gpu/profile.sh CFG [TOP_KERNEL_REGEX] [SKIP]
# 1. launch list: every launch of one warm factorization with its device time;
# 2. per-launch DRAM traffic -> gpurun_out/ncu_traffic_CFG.json (bench.py roofline "traffic");
# 3. one `ncu --set full` capture of the top kernel (SKIP launches of it skipped).
cfg=${1:-c5}; top=${2:-k_update_t}; skip=${3:-100}
mkdir -p gpurun_out
ncu --metrics gpu__time_duration.sum --clock-control none --profile-from-start off --csv \
    --log-file gpurun_out/${cfg}_launches.csv python tools/prof_factor.py $cfg > gpurun_out/${cfg}_launches.log 2>&1
tail -1 gpurun_out/${cfg}_launches.log
ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none \
    --profile-from-start off --csv --log-file gpurun_out/${cfg}_traffic.csv python tools/prof_factor.py $cfg \
    > gpurun_out/${cfg}_traffic.log 2>&1
python tools/ncu_traffic_json.py gpurun_out/${cfg}_traffic.csv $cfg > /dev/null && cp profiles/ncu_traffic_${cfg}.json gpurun_out/
ncu --set full --clock-control none --import-source on --profile-from-start off -k regex:$top -s $skip -c 1 \
    -o gpurun_out/${cfg}_full_${top} python tools/prof_factor.py $cfg > gpurun_out/${cfg}_full.log 2>&1
tail -1 gpurun_out/${cfg}_full.log
