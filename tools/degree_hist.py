"""Degree-bucket histogram of an R-MAT graph (vertices and edges per dispatch class)."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch, graphgen
scale = int(sys.argv[1]) if len(sys.argv) > 1 else 27
dg = graphgen.rmat(scale, seed=1, device=True)
deg = (dg.rowptr[1:] - dg.rowptr[:-1])
edges = [1, 4, 8, 16, 32, 84, 319, 4095, 12287, 1 << 40]
print(f"n={dg.n} nnz={dg.nnz} maxdeg={int(deg.max())}")
lo = 0
for hi in edges[1:]:
    m = (deg > lo) & (deg <= hi)
    print(f"({lo},{hi}]: verts={int(m.sum())} edges={int(deg[m].sum())} frac_edges={float(deg[m].sum())/dg.nnz:.3f}")
    lo = hi
