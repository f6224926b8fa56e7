timeout 300 ./tools/ubench/update_variants 8192 4096 2>&1 | head -6
timeout 300 ./tools/ubench/update_variants 4096 1024 2>&1 | head -6
