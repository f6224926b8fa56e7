./tools/ubench/panel_bench 14900 14900 4
./tools/ubench/panel_bench 4000 4000 4
