# ncu --set full of one dataflow-panel launch on the c5 root (the chain the round-1 verdict named):
# DMMA pipe activity, stall reasons; skip the first $1 (default 170: the root level) panel launches
ncu --set full --clock-control none --import-source on --profile-from-start off -k regex:k_panel -s ${1:-170} -c 1 \
    -o gpurun_out/c5_full_k_panel python tools/prof_factor.py c5 > gpurun_out/c5_panel_full.log 2>&1
tail -2 gpurun_out/c5_panel_full.log
