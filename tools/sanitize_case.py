"""Small factorizations + solves for compute-sanitizer (tools/gpu/sanitize.sh).
Each case checks its factor against the oracle so a silent corruption fails too."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402

import oracle  # noqa: E402
import paper_conf_ipps_georgesgsc11_b200 as mf  # noqa: E402
from tests._grids import grid  # noqa: E402
from tests._parity import ParityStats  # noqa: E402
from workloads import grids as G  # noqa: E402

case = sys.argv[1]
if case == "c1":
    A, p = grid("5pt", (32, 32, 1))
    opts = {}
elif case in ("tiled", "tiled_bulk"):
    A, p = grid("27pt", (16, 16, 16))
    opts = dict(small_front_max=8, variant_model=None)
elif case == "ozaki":
    os.environ["MF_OZ_MIN_K"] = "64"
    A, p = grid("27pt", (16, 16, 16))
    opts = dict(small_front_max=8, variant_model=None, ozaki_slices=8)
else:
    raise SystemExit(f"unknown case {case}")
S = mf.Solver(**opts)
S.analyze(A.n, A.colptr, A.rowind, p)
for _ in range(2):
    S.factor(A.values)
x = S.solve(np.ones(A.n))
sym = oracle.symbolic(A, p)
st = ParityStats()
for s, Po in oracle.factor_stream(A, sym):
    st.add(s, S.panel(s, *Po.shape), Po)
rep = st.report()
print(case, rep)
assert rep["floored_max"] <= 1e-10
print("ok", case, "launches", S.info()["launches_factor"])
