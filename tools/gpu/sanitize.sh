#!/bin/bash
# compute-sanitizer memcheck / racecheck / synccheck over small factorizations that
# reach every kernel family (tools/sanitize_case.py): c1, a 16^3 27-point grid with
# the tiled path forced (dataflow panels, leaves, DMMA updates) with the bulk-copy
# (mbarrier) staging forced on every update (tiled_bulk) or off (tiled: per-thread
# cp.async + CTA barriers), and an Ozaki (int8 tcgen05) run.
mkdir -p gpurun_out
for tool in memcheck racecheck synccheck; do
  for case in c1 tiled tiled_bulk ozaki; do
    env MF_UPD_BULK=$([ $case = tiled_bulk ] && echo 1 || ([ $case = tiled ] && echo 0 || echo -1)) \
      timeout 1200 compute-sanitizer --tool $tool --error-exitcode 9 --print-limit 20 \
      python tools/sanitize_case.py $case > gpurun_out/sanitize_${tool}_${case}.log 2>&1
    echo "$tool $case rc=$? $(grep -E 'ERROR SUMMARY|RACECHECK SUMMARY' gpurun_out/sanitize_${tool}_${case}.log | tail -1)"
  done
done
