timeout 300 ./tools/ubench/update_variants 8192 4096 2>&1 | head -9
