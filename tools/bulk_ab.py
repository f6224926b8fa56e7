"""A/B check of the DMMA update's two staging variants on a config: factor with
MF_UPD_BULK=0 (cp.async) and =1 (bulk copies + mbarriers) in separate
subprocesses, dump per-supernode panel checksums, report the first mismatches."""
import os, subprocess, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np

cfg = sys.argv[1] if len(sys.argv) > 1 else "c5"
if len(sys.argv) > 2 and sys.argv[2] == "child":
    import torch
    import paper_conf_ipps_georgesgsc11_b200 as mf
    from workloads import grids as G
    c = G.CONFIGS[cfg]
    A, p = G.make_config(c["kind"], c["N"])
    nb = int(os.environ.get("NB", "4"))
    S = mf.Solver(nbranch=nb)
    S.analyze(A.n, A.colptr, A.rowind, p)
    S.factor(torch.from_numpy(A.values).cuda())
    sn = S.supernodes()
    k = np.diff(sn["sn_first"]); f = np.diff(sn["sn_rowptr"])
    inf = S.info()
    ld = f + (f & 1)
    tot = int(np.sum(ld * k)) + 2
    Lx = S.export_panels(tot)
    off = np.concatenate([[0], np.cumsum(ld * k)])
    sums = np.array([np.abs(Lx[off[s]:off[s + 1]]).sum() for s in range(len(k))])
    import hashlib
    h = np.array([int.from_bytes(hashlib.md5(Lx[off[s]:off[s + 1]].tobytes()).digest()[:8], "little", signed=True)
                  for s in range(len(k))], dtype=np.int64)
    np.savez(sys.argv[3], sums=sums, h=h, k=k, f=f, par=sn["sn_parent"])
    sys.exit(0)
outs = []
modes = sys.argv[2].split(",") if len(sys.argv) > 2 else ["0", "1"]
for v in modes:
    fn = f"/tmp/bulk_ab_{cfg}_{len(outs)}.npz"
    env = dict(os.environ, MF_UPD_BULK=v.split("r")[0])
    subprocess.run([sys.executable, __file__, cfg, "child", fn], env=env, check=True)
    outs.append(np.load(fn))
a = outs[0]
for v, b in zip(modes[1:], outs[1:]):
    bad = np.nonzero(a["h"] != b["h"])[0]
    print(cfg, "mode", modes[0], "vs", v, "supernodes", len(a["h"]), "mismatching", len(bad), "first", bad[:8])
bad = np.nonzero(a["h"] != outs[-1]["h"])[0]
b = outs[-1]
for s in bad[:6]:
    print(" s", s, "k", a["k"][s], "f", a["f"][s], "parent", a["par"][s], "abs-sum", a["sums"][s], b["sums"][s])
big = np.argsort(-a["f"])[:10]
print("largest fronts:", [(int(s), int(a["k"][s]), int(a["f"][s]), bool(a["h"][s] == b["h"][s])) for s in big])
