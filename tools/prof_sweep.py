"""Profiling driver: generate an R-MAT graph on the device, then run exactly the
kernels to be profiled (no timing claims; use under ncu).

    python tools/prof_sweep.py --scale 27 --what sweep1|run|contract
"""
import argparse
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import graphgen  # noqa: E402
import paper_conf_ipps_naimmht17_b200 as lvb  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--scale", type=int, default=27)
    ap.add_argument("--what", default="sweep1")
    ap.add_argument("--sweeps", type=int, default=1)
    a = ap.parse_args()
    dg = graphgen.rmat(a.scale, seed=1, device=True)
    torch.cuda.synchronize()
    g = lvb.Graph.from_csr(dg.rowptr, dg.col, borrow=True)
    p = lvb.params()
    torch.cuda.cudart().cudaProfilerStart()
    if a.what == "sweep1":
        for _ in range(a.sweeps):
            print(g.sweep(p, with_q=False)[0])
    elif a.what == "sweepq":
        for _ in range(a.sweeps):
            print(g.sweep(p, with_q=True)[0])
    elif a.what == "run":
        print(g.run(p, want_labels=False)[2])
    elif a.what == "contract":
        g.sweep(p, with_q=False)
        g2, _ = g.aggregate(with_map=False)
        print(g2.info())
    torch.cuda.synchronize()
    torch.cuda.cudart().cudaProfilerStop()


if __name__ == "__main__":
    main()
