import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch, graphgen
dg = graphgen.rmat(int(sys.argv[1]) if len(sys.argv) > 1 else 27, seed=1, device=True)
deg = (dg.rowptr[1:] - dg.rowptr[:-1])
edges = [4096, 12288, 32768, 65536, 131072, 262144, 524288, 1 << 40]
lo = edges[0]
for hi in edges[1:]:
    m = (deg >= lo) & (deg < hi)
    print(f"[{lo},{hi}): verts={int(m.sum())} edges={int(deg[m].sum())}")
    lo = hi
