"""Time the oracle on the GPU box's host (SURVEY 8(d) "How the oracle is timed beside it"):
single-threaded plain C, pinned to one core (sched_setaffinity), wall clock of
  * level-0 sweep 1 of oracle (b) (one Alg. 1 repeat body from singletons),
  * phase 1 of oracle (b) (level 0 until its stop test: max_levels = 1),
  * the end-to-end run of oracle (b) (all levels) -- optional, --full,
with `nproc` and the CPU model.  Reported baseline only (not a target).

    python tools/oracle_timing.py C5 [--full] > gpurun_out/oracle_timing_C5.json
"""
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import graphgen  # noqa: E402
import oracle  # noqa: E402


def main():
    cfg = sys.argv[1]
    full = "--full" in sys.argv
    t0 = time.perf_counter()
    try:
        g = graphgen.config(cfg, device=True).to_host()
    except Exception:  # host generator (LFR, karate) or no GPU
        g = graphgen.config(cfg)
    gen_s = time.perf_counter() - t0
    core = max(os.sched_getaffinity(0))
    os.sched_setaffinity(0, {core})
    model = next((ln.split(":", 1)[1].strip() for ln in open("/proc/cpuinfo") if ln.startswith("model name")), None)
    out = {"config": cfg, "n": g.n, "nnz": g.nnz, "gen_s": gen_s, "pinned_core": core, "nproc": os.cpu_count(),
           "cpu_model": model, "oracle": "oracle (b), plain single-threaded C (oracle/louvain_oracle.c)"}
    st = oracle.State(g)
    t0 = time.perf_counter()
    moved = st.sweep(oracle.params())
    out["sweep1_s"] = time.perf_counter() - t0
    out["sweep1_moved"] = moved
    out["sweep1_edges_per_s"] = g.nnz / out["sweep1_s"]
    del st
    t0 = time.perf_counter()
    r = oracle.louvain(g, oracle.params(max_levels=1))
    out["phase1_s"] = time.perf_counter() - t0
    out["phase1_sweeps"] = r.sweeps_per_level[0]
    out["phase1_teps_2E"] = r.sweeps_per_level[0] * g.nnz / out["phase1_s"]
    if full:
        t0 = time.perf_counter()
        r = oracle.louvain(g)
        out["end_to_end_s"] = time.perf_counter() - t0
        out["levels"] = r.levels
        out["q"] = r.q
    print(json.dumps(out), flush=True)


if __name__ == "__main__":
    main()
