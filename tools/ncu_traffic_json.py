"""Per-kernel-class DRAM traffic and device time of ONE warm factorization from an
ncu CSV (gpu__time_duration.sum, dram__bytes_read.sum, dram__bytes_write.sum over
every launch; tools/gpu/profile.sh), joined with the static program's launch
counts and algorithmic bytes -> profiles/ncu_traffic_<cfg>.json, read by bench.py
for the roofline "traffic" field (refused there if the launch count differs from
the benched program).   python tools/ncu_traffic_json.py traffic.csv c5"""
import collections
import csv
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

# kernel (template) base name -> the library's kernel class (mf_kernel_stat names)
CLASS = {"k_update_t": "dmma_schur_update", "k_oz_gemm": "dmma_schur_update", "k_oz_split": "dmma_schur_update",
         "k_oz_rowexp": "dmma_schur_update", "k_assemble": "assemble_extend_add", "k_panel": "dataflow_panel",
         "k_small_front": "small_front_fused", "k_tiny_fronts": "small_front_fused", "k_leaf": "leaf_potrf_trsm",
         "k_potrf_diag": "potrf_diag", "k_trsm_panel": "trsm_panel"}
KIND = {"small_front_fused": 0, "assemble_extend_add": 1, "potrf_diag": 2, "trsm_panel": 3, "dmma_schur_update": 4,
        "leaf_potrf_trsm": 5, "dataflow_panel": 6}
SCALE = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "KB": 1e3, "MB": 1e6, "GB": 1e9, "ns": 1e-9, "us": 1e-6,
         "ms": 1e-3,
         "nsecond": 1e-9, "usecond": 1e-6, "msecond": 1e-3, "second": 1.0}

csv_path, cfg = sys.argv[1], (sys.argv[2] if len(sys.argv) > 2 else "c5")
rows = list(csv.reader(open(csv_path)))
h = None
per = collections.defaultdict(dict)   # launch id -> metrics
name_of = {}
for r in rows:
    if "Kernel Name" in r:
        h = r
        continue
    if h is None or len(r) != len(h):
        continue
    d = dict(zip(h, r))
    base = d["Kernel Name"].split("(")[0].split("<")[0].replace("void ", "").replace("mf::", "").strip()
    name_of[d["ID"]] = base
    per[d["ID"]][d["Metric Name"]] = float(d["Metric Value"].replace(",", "")) * SCALE.get(d["Metric Unit"], 1)

import paper_conf_ipps_georgesgsc11_b200 as mf  # noqa: E402
from workloads import grids as G  # noqa: E402
c = G.CONFIGS[cfg]
A, p = G.make_config(c["kind"], c["N"])
S = mf.Solver(host_only=True)
S.analyze(A.n, A.colptr, A.rowind, p)
prog = S.program()

out = {"config": cfg, "program_launches": len(prog), "kernels": {}}
tot_time = sum(m.get("gpu__time_duration.sum", 0.0) for m in per.values())
for cls, kind in KIND.items():
    ids = [i for i, b in name_of.items() if CLASS.get(b) == cls and b not in ("k_oz_split", "k_oz_rowexp")]
    if not ids:
        continue
    byts = [per[i].get("dram__bytes_read.sum", 0) + per[i].get("dram__bytes_write.sum", 0) for i in ids]
    t = [per[i].get("gpu__time_duration.sum", 0.0) for i in ids]
    algo = [L["bytes"] for L in prog if L["kind"] == kind]
    e = {"launches": len(ids), "program_launches": len(algo),
         "dram_bytes_per_launch": sum(byts) / len(byts),
         "ncu_time_ms": sum(t) * 1e3, "share_of_ncu_time": sum(t) / tot_time if tot_time else None,
         "dram_GBps_ncu": sum(byts) / sum(t) / 1e9 if sum(t) else None}
    if algo:
        e["algorithmic_bytes_per_launch"] = sum(algo) / len(algo)
        e["algorithmic_GBps_ncu"] = sum(algo) / sum(t) / 1e9 if sum(t) else None
        e["traffic_over_algorithmic"] = (sum(byts) / sum(algo)) if sum(algo) else None
    out["kernels"][cls] = e
out["_source"] = (f"ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum "
                  f"--clock-control none over every launch of one warm {cfg} factorization "
                  "(cold-cache, serialised replays: compare shares, not absolute times)")
dst = os.path.join(ROOT, "profiles", f"ncu_traffic_{cfg}.json")
json.dump(out, open(dst, "w"), indent=1)
print(json.dumps(out, indent=1))
