"""Time one louvain_sweep (sweep 1 from singletons) with CUDA events; repeat R times."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch, graphgen
import paper_conf_ipps_naimmht17_b200 as lvb
scale = int(sys.argv[1]) if len(sys.argv) > 1 else 27
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 3
dg = graphgen.rmat(scale, seed=1, device=True)
s = torch.cuda.Stream()
g = lvb.Graph.from_csr(dg.rowptr, dg.col, borrow=True, stream=s)
p = lvb.params()
ts = []
for r in range(reps + 1):
    g.set_labels(None)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(s)
    mv, _ = g.sweep(p, with_q=False)
    e1.record(s)
    torch.cuda.synchronize()
    if r: ts.append(e0.elapsed_time(e1))
print(f"{os.environ.get('TAG','')} sweep1 ms: {min(ts):.2f} (moved {mv})")
