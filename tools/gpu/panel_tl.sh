# dataflow-panel phase timeline (tools/ubench/panel_timeline.cu): new vs old potrf, bitwise hash
for b in panel_timeline panel_timeline_old; do for a in "6545 6545 8" "15000 15000 8" "2000 1000 8" "1000 700 8" "333 250 8"; do echo "== $b $a"; timeout 60 ./tools/ubench/$b $a | grep -v "^row" | grep -E "^f=|hash|max|potrf steps|^band (0|3|7)"; done; done > gpurun_out/panel_tl3.txt 2>&1
