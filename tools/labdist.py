import os, sys
sys.path.insert(0, '/root/repo')
import torch, graphgen, numpy as np
import paper_conf_ipps_naimmht17_b200 as lvb
dg = graphgen.rmat(27, seed=1, device=True)
g = lvb.Graph.from_csr(dg.rowptr, dg.col, borrow=True)
p = lvb.params()
# after buckets 1-6 commit, what labels do hub neighbours carry?  emulate: run a sweep with bounds making
# bucket 7 empty, i.e. deg_bounds[5] huge -> all non-hub... simpler: run one full sweep and inspect labels
g.sweep(p, with_q=False)
lab = torch.empty(dg.n, dtype=torch.int32, device='cuda'); g.labels(lab)
deg = dg.rowptr[1:] - dg.rowptr[:-1]
hubs = torch.nonzero(deg >= 12288).flatten()
tot = 0; same_own = 0; top1 = 0
for h in hubs[:200].tolist():
    nb = dg.col[dg.rowptr[h]:dg.rowptr[h+1]].long()
    l = lab[nb]
    vals, cnt = torch.unique(l, return_counts=True)
    tot += nb.numel(); top1 += int(cnt.max()); same_own += int((l == h).sum())
print('first 200 hubs: edges', tot, 'top-label share', top1 / tot, 'label==hub share', same_own / tot)
