# graph node priorities for the chain kernels (MF_NODE_PRIO): factor times c2-c5 + targeted tests
timeout 900 python -m pytest tests -m gpu -q -x -k "manufactured or lookahead or variant or parity_small or bulk" > gpurun_out/prio_test.log 2>&1; tail -1 gpurun_out/prio_test.log
for e in 0 1; do MF_NODE_PRIO=$e timeout 900 python tools/time_factor.py c2 c3 c4 c5; done > gpurun_out/prio_ab.txt 2>&1; cat gpurun_out/prio_ab.txt
