# panel width A/B (kPanelMaxBlocks builds under build/ab/): factor times c2 / c3 / c5
for nb in 8 6 12; do cp build/ab/libmf_nb$nb.so paper_conf_ipps_georgesgsc11_b200/libmf.so; touch paper_conf_ipps_georgesgsc11_b200/libmf.so
  timeout 900 python tools/time_factor.py c2 c3 c5 | sed "s/^/nbk=$nb /"; done > gpurun_out/nbk_ab.txt 2>&1
cp build/ab/libmf_nb8.so paper_conf_ipps_georgesgsc11_b200/libmf.so
