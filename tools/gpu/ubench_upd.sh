set -x
timeout 300 ./tools/ubench/update_variants 8192 4096 > gpurun_out/ubench_upd.txt 2>&1; cat gpurun_out/ubench_upd.txt
timeout 300 ./tools/ubench/update_variants 4096 1024 > gpurun_out/ubench_upd2.txt 2>&1; cat gpurun_out/ubench_upd2.txt
