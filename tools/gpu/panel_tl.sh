# dataflow-panel phase timeline (tools/ubench/panel_timeline.cu, built with the PANEL_TL hook) + fp64 latency / potrf part ubenches
for a in "6545 6545 8" "15000 15000 8" "2000 1000 8"; do ./tools/ubench/panel_timeline $a | grep -v "^row"; done > gpurun_out/panel_tl.txt 2>&1
./tools/ubench/lat >> gpurun_out/panel_tl.txt 2>&1
./tools/ubench/potrf_parts >> gpurun_out/panel_tl.txt 2>&1
