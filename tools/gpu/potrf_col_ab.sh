# potrf trailing update by block column: bitwise hash of c2-c4 L, panel timeline, factor times, targeted tests
python - > gpurun_out/hash_new.txt 2>&1 <<PY
import sys, hashlib
sys.path.insert(0, ".")
import numpy as np
import paper_conf_ipps_georgesgsc11_b200 as mf
from workloads import grids as G
for cfg in ("c2", "c3", "c4"):
    c = G.CONFIGS[cfg]
    A, p = G.make_config(c["kind"], c["N"])
    S = mf.Solver(); S.analyze(A.n, A.colptr, A.rowind, p); S.factor(A.values)
    Lp, Li, Lx = S.export_L()
    print(cfg, hashlib.sha256(np.ascontiguousarray(Lx).tobytes()).hexdigest()[:16])
PY
cat gpurun_out/hash_new.txt
for a in "6545 6545 8" "15000 15000 8"; do ./tools/ubench/panel_timeline $a | grep -E "^f=|^band 7"; done > gpurun_out/potrf_col_tl.txt 2>&1
timeout 900 python tools/time_factor.py c2 c3 c4 c5 > gpurun_out/potrf_col_ab.txt 2>&1; cat gpurun_out/potrf_col_ab.txt
timeout 600 python tools/dense_potrf.py 7014 14900 >> gpurun_out/potrf_col_ab.txt 2>&1
timeout 1200 python -m pytest tests -m gpu -q -x -k "manufactured or parity or variant or lookahead or dense or not_spd" > gpurun_out/potrf_col_test.log 2>&1; tail -1 gpurun_out/potrf_col_test.log
