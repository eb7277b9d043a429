"""Where the end-to-end time goes (C5): pinned H2D bandwidth, louvain_create_csr from
host buffers, run, labels D2H.  Diagnostics only (no bench claims)."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch, graphgen
import paper_conf_ipps_naimmht17_b200 as lvb
dg = graphgen.rmat(int(sys.argv[1]) if len(sys.argv) > 1 else 27, seed=1, device=True)
n, nnz = dg.n, dg.nnz
h_rowptr = torch.empty(n + 1, dtype=torch.int64, pin_memory=True); h_rowptr.copy_(dg.rowptr)
h_col = torch.empty(nnz, dtype=torch.int32, pin_memory=True); h_col.copy_(dg.col)
h_lab = torch.empty(n, dtype=torch.int32, pin_memory=True)
d = torch.empty(nnz, dtype=torch.int32, device="cuda")
for _ in range(2):
    torch.cuda.synchronize(); t = time.perf_counter(); d.copy_(h_col, non_blocking=True); torch.cuda.synchronize()
    print(f"torch H2D {4*nnz/1e9:.2f} GB: {(time.perf_counter()-t)*1e3:.1f} ms = {4*nnz/1e9/(time.perf_counter()-t):.1f} GB/s", flush=True)
del d
g0 = lvb.Graph.from_csr(dg.rowptr, dg.col, borrow=True); g0.run(lvb.params(), labels_out=h_lab); del g0
del dg; torch.cuda.empty_cache()
p = lvb.params()
for r in range(3):
    torch.cuda.synchronize(); t0 = time.perf_counter()
    g = lvb.Graph.from_csr(h_rowptr, h_col)
    torch.cuda.synchronize(); t1 = time.perf_counter()
    g.run(p, labels_out=h_lab)
    torch.cuda.synchronize(); t2 = time.perf_counter()
    g.close()
    torch.cuda.synchronize(); t3 = time.perf_counter()
    print(f"e2e {r}: create {1e3*(t1-t0):.1f} ms, run+D2H {1e3*(t2-t1):.1f} ms, close {1e3*(t3-t2):.1f} ms", flush=True)
