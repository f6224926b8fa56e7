# concurrent-graph timelines (tools/timeline.py) of c2 / c3 / c5 + the ABI / profiling tests
timeout 600 python -m pytest tests -m gpu -q -x -k "profil or abi or stats" > gpurun_out/tl_test.log 2>&1; tail -1 gpurun_out/tl_test.log
for c in c2 c3 c5; do timeout 600 python tools/timeline.py $c --csv gpurun_out/timeline_$c.csv > gpurun_out/timeline_$c.txt 2>&1; head -12 gpurun_out/timeline_$c.txt; done
