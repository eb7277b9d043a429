"""Experiment (performance only, not semantics): level-0 sweep-1 time of C5 in
the generator's id order vs. after relabelling the vertices by degree
(descending), with and without a persisting L2 window over the hot prefix of
the vertex records (LV_L2WIN).  Relabelling changes tie-breaks, so the moved
counts differ; only the times are compared.

    LV_TRACE=2 python tools/relabel_exp.py --scale 27
"""
import argparse
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def relabel(rowptr, col, chunk=1 << 28):
    import torch
    n = rowptr.numel() - 1
    deg = rowptr[1:] - rowptr[:-1]
    order = torch.sort(deg, descending=True, stable=True).indices  # new -> old
    pi = torch.empty_like(order)
    pi[order] = torch.arange(n, device=order.device)
    pi32 = pi.to(torch.int32)
    deg_new = deg[order]
    rp_new = torch.zeros(n + 1, dtype=torch.int64, device=rowptr.device)
    torch.cumsum(deg_new, 0, out=rp_new[1:])
    shift = rowptr[:-1][order] - rp_new[:-1]  # src = dst + shift(row)
    nnz = int(rp_new[-1])
    col_new = torch.empty(nnz, dtype=torch.int32, device=col.device)
    # rows are cut into chunks of ~chunk entries
    r0 = 0
    while r0 < n:
        e0 = int(rp_new[r0])
        r1 = int(torch.searchsorted(rp_new, min(e0 + chunk, nnz), right=False))
        r1 = max(r1, r0 + 1)
        r1 = min(r1, n)
        e1 = int(rp_new[r1])
        sh = torch.repeat_interleave(shift[r0:r1], deg_new[r0:r1], output_size=e1 - e0)
        src = torch.arange(e0, e1, device=col.device, dtype=torch.int64) + sh
        col_new[e0:e1] = pi32[col[src].long()]
        del sh, src
        r0 = r1
    return rp_new, col_new


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--scale", type=int, default=27)
    ap.add_argument("--mode", default="both")
    a = ap.parse_args()
    import torch
    import graphgen
    import paper_conf_ipps_naimmht17_b200 as lvb
    dg = graphgen.rmat(a.scale, seed=1, device=True)
    torch.cuda.synchronize()
    rp, cl = dg.rowptr, dg.col
    if a.mode in ("relabel", "both"):
        rp2, cl2 = relabel(rp, cl)
        torch.cuda.synchronize()
        if a.mode == "relabel":
            del dg
            rp, cl = rp2, cl2
    for name, (r, c) in ([("natural", (rp, cl))] if a.mode == "natural" else []) + \
            ([("relabel", (rp2, cl2))] if a.mode in ("relabel", "both") else []) + \
            ([("natural", (dg.rowptr, dg.col))] if a.mode == "both" else []):
        for rep in range(2):
            g = lvb.Graph.from_csr(r, c, borrow=True)
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            print(f"==== {name} rep {rep}", file=sys.stderr, flush=True)
            e0.record()
            moved = g.sweep(lvb.params(), with_q=False)[0]
            e1.record()
            torch.cuda.synchronize()
            print(f"{name} rep {rep}: moved {moved} sweep+binning {e0.elapsed_time(e1):.2f} ms", flush=True)
            g.close()


if __name__ == "__main__":
    main()
