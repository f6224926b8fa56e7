./tools/ubench/update_trap 16 3000 256 256 30
./tools/ubench/update_trap 30 2000 128 128 30
./tools/ubench/update_trap 8 4000 512 512 20
timeout 300 ./tools/ubench/update_variants 8192 4096 2>&1 | head -4
timeout 300 ./tools/ubench/update_variants 4096 1024 2>&1 | head -4
