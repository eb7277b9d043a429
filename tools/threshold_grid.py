"""NEXT-4: threshold-grid replay of the GPU path on the BASELINE configs.

The paper's Figs. 1-2 and 4 vary the phase threshold used while n > 100,000
(theta_bin) and the one used on small levels (theta_final).  This replays that grid on our
synthetic workloads through `louvain_run` (the GPU path, bit-identical to oracle (b) at every
setting -- tests/test_gpu_parity.py::test_full_run_threshold_grid), one JSON line per
(config, th_bin_exp, th_final_exp): Q, levels, sweeps, edges swept, run time (CUDA events on the
handle's stream, median of 3 after one warm-up run).

  python tools/threshold_grid.py [C2 C3 C4a C4b C5]
"""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import graphgen  # noqa: E402
import paper_conf_ipps_naimmht17_b200 as lvb  # noqa: E402

CONFIGS = {
    "C2": lambda: graphgen.lfr(1_000_000, seed=1),
    "C3": lambda: graphgen.rmat(24, seed=1, device=True),
    "C4a": lambda: graphgen.mesh3d(368, True, device=True),
    "C4b": lambda: graphgen.rgg(50_000_000, seed=1, device=True),
    "C5": lambda: graphgen.rmat(27, seed=1, device=True),
}
TH_BIN = (1, 2, 3, 4)        # theta_bin = 10^-e while n_level > size_limit (paper default e = 2)
TH_FINAL = (3, 4, 6, 7)      # theta_final = 10^-e on small levels and the level test (default 6)


def main():
    names = sys.argv[1:] or list(CONFIGS)
    for name in names:
        g0 = CONFIGS[name]()
        stream = torch.cuda.Stream()
        if isinstance(g0.rowptr, torch.Tensor):
            g = lvb.Graph.from_csr(g0.rowptr, g0.col, borrow=True, stream=stream)
        else:
            g = lvb.Graph.from_csr(g0.rowptr, g0.col, g0.w, stream=stream)
        for tb in TH_BIN:
            for tf in TH_FINAL:
                p = lvb.params(th_bin_exp=tb, th_final_exp=tf)
                g.run(p, want_labels=False)
                ms, out = [], None
                for _ in range(3):
                    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                    e0.record(stream)
                    _, q, st = g.run(p, want_labels=False)
                    e1.record(stream)
                    e1.synchronize()
                    ms.append(e0.elapsed_time(e1))
                    out = (q, st)
                q, st = out
                print(json.dumps({"config": name, "th_bin_exp": tb, "th_final_exp": tf, "q": q.q,
                                  "levels": st["levels"], "sweeps": sum(st["sweeps_per_level"]),
                                  "sweeps_per_level": st["sweeps_per_level"],
                                  "edges_swept": st["edges_swept"], "ms": sorted(ms)[1],
                                  "default": (tb, tf) == (2, 6)}), flush=True)
        del g
        torch.cuda.empty_cache()


if __name__ == "__main__":
    t = time.time()
    main()
    print(json.dumps({"wall_s": time.time() - t}), file=sys.stderr)
