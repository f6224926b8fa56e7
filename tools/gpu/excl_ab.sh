# band-SM exclusion of the dataflow panel: timeline ubench + factor A/B + targeted tests
for a in "15000 15000 8 0" "15000 15000 8 8" "8192 8192 8 0" "8192 8192 8 8" "6545 6545 8 8"; do ./tools/ubench/panel_timeline $a | grep -v "^row"; done > gpurun_out/excl_tl.txt 2>&1
for e in 0 1 2; do MF_PANEL_EXCL=$e timeout 600 python tools/time_factor.py c2 c3 c5; done > gpurun_out/excl_ab.txt 2>&1
MF_PANEL_EXCL=2 timeout 900 python -m pytest tests -m gpu -q -x -k "panel or manufactured or parity" > gpurun_out/excl_test.log 2>&1; tail -2 gpurun_out/excl_test.log
