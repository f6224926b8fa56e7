# A/B of the dataflow-solve register ring (MF_DF_VARIANT) on c5 and c3
for v in 0 1 2 3; do for c in c5 c3; do echo "variant $v: $(MF_DF_VARIANT=$v timeout 300 python tools/solve_time.py $c)"; done; done > gpurun_out/df_variants.txt 2>&1
cat gpurun_out/df_variants.txt
