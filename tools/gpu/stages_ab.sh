# dataflow-panel operand ring A/B (MF_PANEL_STAGES / MF_PANEL_MINB builds under build/ab/): c2 / c3 / c5 times
for v in nb8 st3_mb2 st3_mb1; do cp build/ab/libmf_$v.so paper_conf_ipps_georgesgsc11_b200/libmf.so; touch paper_conf_ipps_georgesgsc11_b200/libmf.so
  timeout 900 python tools/time_factor.py c2 c3 c5 | sed "s/^/$v /"; done > gpurun_out/stages_ab.txt 2>&1
cp build/ab/libmf_nb8.so paper_conf_ipps_georgesgsc11_b200/libmf.so
