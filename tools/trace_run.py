import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
os.environ.setdefault("LV_TRACE", "1")
import torch, graphgen
import paper_conf_ipps_naimmht17_b200 as lvb
dg = graphgen.rmat(int(sys.argv[1]) if len(sys.argv) > 1 else 27, seed=1, device=True)
s = torch.cuda.Stream()
g = lvb.Graph.from_csr(dg.rowptr, dg.col, borrow=True, stream=s)
for r in range(2):
    print(f"---- run {r}", file=sys.stderr, flush=True)
    lab, q, st = g.run(lvb.params(), want_labels=False)
