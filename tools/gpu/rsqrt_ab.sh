# pivot rsqrt with one second-order refinement: factor tests (manufactured bit-exact, parity, full-tree c2/c3) + times + hash
timeout 1500 python -m pytest tests -m gpu -q -x -k "manufactured or parity or variant or nanfill or lookahead or bulk or fulltree and (c2 or c3) or dense or not_spd or loopback_manufactured" > gpurun_out/rsqrt_test.log 2>&1; tail -1 gpurun_out/rsqrt_test.log
timeout 900 python tools/time_factor.py c2 c3 c4 c5 > gpurun_out/rsqrt_ab.txt 2>&1; cat gpurun_out/rsqrt_ab.txt
timeout 600 python tools/dense_potrf.py 7014 5418 >> gpurun_out/rsqrt_ab.txt 2>&1; tail -2 gpurun_out/rsqrt_ab.txt
