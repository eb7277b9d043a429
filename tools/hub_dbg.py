import os, sys, ctypes
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
os.environ["LV_DEBUG_HUB"] = os.environ.get("LV_DEBUG_HUB", "256")
import torch, graphgen
import paper_conf_ipps_naimmht17_b200 as lvb
dg = graphgen.rmat(27, seed=1, device=True)
g = lvb.Graph.from_csr(dg.rowptr, dg.col, borrow=True)
p = lvb.params()
L = lvb.lib()
out = (ctypes.c_ulonglong * 8)()
g.set_labels(None); g.sweep(p, with_q=False); L.lv_debug_hub(out, 1)
for r in range(2):
    g.set_labels(None)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(); g.sweep(p, with_q=False); e1.record(); torch.cuda.synchronize()
    L.lv_debug_hub(out, 1)
    cyc = 1.965e9
    print(f"sweep {e0.elapsed_time(e1):.1f} ms; CTA-seconds wait {out[0]/cyc:.3f} insert {out[1]/cyc:.3f} scan {out[2]/cyc:.3f}; items ins {out[4]} scan {out[5]}")
