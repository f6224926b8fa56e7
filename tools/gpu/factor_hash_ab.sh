# factor A/B driver: bitwise hash of c2 / c3 L (export_L), targeted factor tests, c2 / c3 / c5 times
python - > gpurun_out/factor_hash.txt 2>&1 <<'PY'
import sys, hashlib
sys.path.insert(0, ".")
import numpy as np
import paper_conf_ipps_georgesgsc11_b200 as mf
from workloads import grids as G
for cfg in ("c2", "c3"):
    c = G.CONFIGS[cfg]
    A, p = G.make_config(c["kind"], c["N"])
    S = mf.Solver()
    S.analyze(A.n, A.colptr, A.rowind, p)
    S.factor(A.values)
    Lp, Li, Lx = S.export_L()
    print(cfg, hashlib.sha256(np.ascontiguousarray(Lx).tobytes()).hexdigest()[:16])
PY
cat gpurun_out/factor_hash.txt
timeout 900 python -m pytest tests -m gpu -q -x -k "fused or manufactured or parity or variant or nanfill or assemble or dup" > gpurun_out/factortest_hash.log 2>&1; tail -1 gpurun_out/factortest_hash.log
timeout 600 python tools/time_factor.py c2 c3 c5 > gpurun_out/factor_hash_ab.txt 2>&1; cat gpurun_out/factor_hash_ab.txt
