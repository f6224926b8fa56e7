# round-1 (session 3) profile set: launch list, per-launch DRAM traffic, full captures
set -x
ncu --metrics gpu__time_duration.sum --clock-control none --profile-from-start off --csv --log-file gpurun_out/c5_launches_s3.csv python tools/prof_factor.py c5 > gpurun_out/launches.log 2>&1; tail -1 gpurun_out/launches.log
ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --profile-from-start off -k regex:"k_update_t|k_assemble|k_panel" --csv --log-file gpurun_out/traffic_c5_s3.csv python tools/prof_factor.py c5 > gpurun_out/traffic.log 2>&1; tail -1 gpurun_out/traffic.log
NB=1 ncu --set full --clock-control none --import-source on --profile-from-start off -k regex:k_update_t -s 43 -c 1 -o gpurun_out/prof_update_s3 python tools/prof_factor.py c5 > gpurun_out/ncu_full.log 2>&1; tail -1 gpurun_out/ncu_full.log
NB=1 ncu --set full --clock-control none --import-source on --profile-from-start off -k regex:k_panel -s 91 -c 1 -o gpurun_out/prof_panel_s3 python tools/prof_factor.py c5 > gpurun_out/ncu_panel.log 2>&1; tail -1 gpurun_out/ncu_panel.log
