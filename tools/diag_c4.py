import numpy as np, sys
sys.path.insert(0, '.')
import oracle
import paper_conf_ipps_georgesgsc11_b200 as mf
from workloads import grids as G
c = G.CONFIGS['c4']; A, p = G.make_config(c['kind'], c['N'])
S = mf.Solver(); S.analyze(A.n, A.colptr, A.rowind, p); S.factor(A.values)
sym = oracle.symbolic(A, p)
ch = sym.children()
sizes = np.zeros(sym.nsuper, dtype=np.int64)
for s in range(sym.nsuper):
    sizes[s] = 1 + sum(sizes[q] for q in ch[s])
picks = [int(np.argmax(np.where(sizes < lim, sizes, 0))) for lim in (40, 400, 3000)]
subset = set()
for r in picks:
    st = [r]
    while st:
        v = st.pop(); subset.add(v); st.extend(ch[v])
panels = oracle.factor(A, sym, subset=subset)
worst = []
for s, Po in panels.items():
    f, k = Po.shape
    Pg = S.panel(s, f, k)
    colmax = np.abs(Po).max(axis=0)
    for tau in (1e-6, 1e-8):
        den = np.maximum(np.abs(Po), tau * colmax[None, :]); den[den == 0] = 1
        rel = np.abs(Pg - Po) / den
        i = np.unravel_index(np.argmax(rel), rel.shape)
        worst.append((tau, rel.max(), s, f, k, abs(Po[i]) / colmax[i[1]], np.abs(Pg - Po).max() / np.abs(Po).max()))
for tau in (1e-6, 1e-8):
    w = max((x for x in worst if x[0] == tau), key=lambda x: x[1])
    print("tau", tau, "worst C11", w[1], "at s,f,k", w[2:5], "entry/colmax", w[5], "panel absmax-rel", w[6])
print("max abs rel (vs panel max):", max(x[6] for x in worst))
