"""Degree histogram of every level of a C5-like run (contracted graphs via the C-ABI)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch, graphgen
import paper_conf_ipps_naimmht17_b200 as lvb
scale = int(sys.argv[1]) if len(sys.argv) > 1 else 27
dg = graphgen.rmat(scale, seed=1, device=True)
g = lvb.Graph.from_csr(dg.rowptr, dg.col, borrow=True)
p = lvb.params()
for level in range(4):
    n, nnz, W = g.info()
    rp = np.empty(n + 1, dtype=np.int64)
    lvb.lib().louvain_get_csr(g._h, rp.ctypes.data, None, None)
    deg = np.diff(rp)
    edges = [0, 32, 340, 1024, 4096, 12288, 32768, 393216, 1 << 40]
    row = []
    for lo, hi in zip(edges[:-1], edges[1:]):
        m = (deg > lo) & (deg <= hi)
        row.append(f"({lo},{hi}]:{int(m.sum())}v/{int(deg[m].sum())/1e6:.1f}Me")
    print(f"level {level}: n={n} nnz={nnz} maxdeg={deg.max()} | " + " ".join(row), flush=True)
    for s in range(2):
        mv, _ = g.sweep(p, with_q=False)
        if mv == 0: break
    g2, _ = g.aggregate(with_map=False)
    g = g2
