"""Per-launch DRAM traffic of the hot kernels from an ncu CSV (dram__bytes_read.sum,
dram__bytes_write.sum over every launch of one warm factorization) joined with the
static program's algorithmic bytes -> profiles/ncu_traffic.json (read by bench.py
for the roofline "traffic" field).   python tools/ncu_traffic_json.py traffic.csv [c5]"""
import collections, csv, json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

NAMES = {"k_update_t": "dmma_schur_update", "k_assemble": "assemble_extend_add", "k_panel": "dataflow_panel",
         "k_small_front": "small_front_fused"}
KIND = {"dmma_schur_update": 4, "assemble_extend_add": 1, "dataflow_panel": 6, "small_front_fused": 0}
scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "KB": 1e3, "MB": 1e6, "GB": 1e9}
rows = list(csv.reader(open(sys.argv[1])))
h = None
per = collections.defaultdict(lambda: collections.defaultdict(float))
for r in rows:
    if "Kernel Name" in r:
        h = r
        continue
    if h is None or len(r) != len(h):
        continue
    d = dict(zip(h, r))
    base = d["Kernel Name"].split("(")[0].split("<")[0].replace("void ", "").replace("mf::", "").strip()
    if base not in NAMES or not d["Metric Name"].startswith("dram__bytes"):
        continue
    per[(NAMES[base], d["ID"])][d["Metric Name"]] += float(d["Metric Value"].replace(",", "")) * scale.get(d["Metric Unit"], 1)
out = {}
cfg = sys.argv[2] if len(sys.argv) > 2 else "c5"
algo = collections.defaultdict(list)
try:
    import paper_conf_ipps_georgesgsc11_b200 as mf
    from workloads import grids as G
    c = G.CONFIGS[cfg]
    A, p = G.make_config(c["kind"], c["N"])
    S = mf.Solver(host_only=True)
    S.analyze(A.n, A.colptr, A.rowind, p)
    for L in S.program():
        algo[L["kind"]].append(L["bytes"])
except Exception as e:  # noqa: BLE001
    print("no algorithmic join:", e)
for name in NAMES.values():
    launches = [v for (n, _), v in per.items() if n == name]
    if not launches:
        continue
    tot = [v.get("dram__bytes_read.sum", 0) + v.get("dram__bytes_write.sum", 0) for v in launches]
    out[name] = sum(tot) / len(tot)
    out[name + "_launches"] = len(tot)
    a = algo.get(KIND[name])
    if a:
        out[name + "_algorithmic_bytes_per_launch"] = sum(a) / len(a)
out["_source"] = (f"ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum over every launch of one warm {cfg} "
                  "factorization (tools/gpu/ncu_traffic.sh); bytes per launch (mean)")
json.dump(out, open(os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "profiles",
                                 "ncu_traffic.json"), "w"), indent=1)
print(json.dumps(out, indent=1))
