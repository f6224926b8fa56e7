"""Element-level diff between MF_UPD_BULK modes (debug tool for the bulk-copy
Schur update): the first mismatching supernode in postorder and where in its
panel the entries differ.   python tools/bulk_diff.py c3 3 [runs]"""
import os, subprocess, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np

cfg, mode = sys.argv[1], sys.argv[2]
if len(sys.argv) > 3 and sys.argv[3] == "child":
    import torch
    import paper_conf_ipps_georgesgsc11_b200 as mf
    from workloads import grids as G
    c = G.CONFIGS[cfg]
    A, p = G.make_config(c["kind"], c["N"])
    S = mf.Solver(nbranch=1)
    S.analyze(A.n, A.colptr, A.rowind, p)
    S.factor(torch.from_numpy(A.values).cuda())
    sn = S.supernodes()
    k = np.diff(sn["sn_first"]); f = np.diff(sn["sn_rowptr"])
    ld = f + (f & 1)
    Lx = S.export_panels(int(np.sum(ld * k)) + 2)
    np.save(sys.argv[4], Lx)
    np.savez(sys.argv[4] + ".meta.npz", k=k, f=f, par=sn["sn_parent"])
    sys.exit(0)
runs = int(sys.argv[3]) if len(sys.argv) > 3 else 4
ref = f"/tmp/bd_{cfg}_ref.npy"
subprocess.run([sys.executable, __file__, cfg, mode, "child", ref], env=dict(os.environ, MF_UPD_BULK="0"), check=True)
R = np.load(ref, mmap_mode="r")
meta = np.load(ref + ".meta.npz")
k, f = meta["k"], meta["f"]
ld = f + (f & 1)
off = np.concatenate([[0], np.cumsum(ld * k)])
for r in range(runs):
    fn = f"/tmp/bd_{cfg}_run.npy"
    subprocess.run([sys.executable, __file__, cfg, mode, "child", fn], env=dict(os.environ, MF_UPD_BULK=mode), check=True)
    B = np.load(fn, mmap_mode="r")
    diff = np.nonzero(np.asarray(R[:off[-1]]) != np.asarray(B[:off[-1]]))[0]
    if diff.size == 0:
        print(f"run {r}: identical", flush=True)
        continue
    sids = np.searchsorted(off, diff, side="right") - 1
    first = int(sids.min())
    print(f"run {r}: {diff.size} words differ in {np.unique(sids).size} supernodes; first s={first} k={k[first]} "
          f"f={f[first]} parent={meta['par'][first]}")
    w = diff[sids == first] - off[first]
    cols, rows = w // ld[first], w % ld[first]
    a = np.asarray(R[off[first]:off[first + 1]]).reshape(k[first], ld[first]).T
    b = np.asarray(B[off[first]:off[first + 1]]).reshape(k[first], ld[first]).T
    print(f"   {w.size} entries; cols {cols.min()}..{cols.max()} rows {rows.min()}..{rows.max()} "
          f"max|diff| {np.abs(a - b).max():.3e}")
    c0 = cols.min()
    print(f"   first col {c0}: rows {rows[cols == c0][:40]}")
    print(f"   cols with diffs: {np.unique(cols)[:40]}")
    print(f"   64-tiles (row//64, col//64): {sorted({(int(x) // 64, int(y) // 64) for x, y in zip(rows, cols)})[:40]}",
          flush=True)
