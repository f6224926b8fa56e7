# full ncu capture of the two largest DMMA update launches of one warm c5 factorization
ncu --set full --clock-control none --import-source on --profile-from-start off -k regex:k_update -s ${1:-103} -c 1 -o gpurun_out/prof_update_big python tools/prof_factor.py c5 > gpurun_out/ncu_big.log 2>&1; tail -2 gpurun_out/ncu_big.log
ncu --set full --clock-control none --import-source on --profile-from-start off -k regex:k_assemble -s 10 -c 1 -o gpurun_out/prof_asm python tools/prof_factor.py c5 > gpurun_out/ncu_asm.log 2>&1; tail -2 gpurun_out/ncu_asm.log
