"""Time louvain_run on one BASELINE config (median of 3 after a warm-up run); prints one JSON
line with the run time and the stats' modularity / sweep / contraction totals.  Used to A/B
environment switches (each process reads them once):  LV_DELTA_DIV=1 python tools/run_time.py C4a"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_ipps_naimmht17_b200 as lvb  # noqa: E402
from tools.threshold_grid import CONFIGS  # noqa: E402

name = sys.argv[1]
g0 = CONFIGS[name]()
stream = torch.cuda.Stream()
if isinstance(g0.rowptr, torch.Tensor):
    g = lvb.Graph.from_csr(g0.rowptr, g0.col, borrow=True, stream=stream)
else:
    g = lvb.Graph.from_csr(g0.rowptr, g0.col, g0.w, stream=stream)
g.run(want_labels=False)
rows = []
for _ in range(3):
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(stream)
    _, q, st = g.run(want_labels=False)
    e1.record(stream)
    e1.synchronize()
    rows.append((e0.elapsed_time(e1), st, q.q))
rows.sort(key=lambda r: r[0])
ms, st, q = rows[1]
print(json.dumps({"config": name, "env": {k: v for k, v in os.environ.items() if k.startswith("LV_")}, "ms": ms,
                  "t_modularity_ms_total": st["t_modularity_ms_total"], "t_sweep_ms_total": st["t_sweep_ms_total"],
                  "sweeps": st["sweeps"], "q": q}), flush=True)
