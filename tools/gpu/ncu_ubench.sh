set -x
./tools/ubench/update_variants 8192 4096 > gpurun_out/ubench_upd.txt 2>&1; cat gpurun_out/ubench_upd.txt
ncu --set full --clock-control none --import-source on -k regex:k_update_t -s 1 -c 1 -o gpurun_out/prof_ubench_upd ./tools/ubench/update_variants 8192 4096 > gpurun_out/ncu_ubench.log 2>&1; tail -2 gpurun_out/ncu_ubench.log
