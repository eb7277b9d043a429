"""BASELINE.md §8 result rows from the round's evidence: bench lines (profiles/r02/final/bench_*.jsonl),
the oracle's golden runs (tests/golden/oracle_runs.json) and the oracle timing on the GPU host
(profiles/r02/r2d_oracle_timing_*.json).

    python tools/results_table.py profiles/r02/final
"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
NAMES = {"C1": "C1 karate", "C2": "C2 LFR 1M", "C3": "C3 R-MAT s24", "C4a": "C4a mesh 368³ (Morton ids)",
         "C4b": "C4b RGG 5e7", "C5": "C5 R-MAT s27"}


def main():
    d = sys.argv[1]
    gold = json.load(open(os.path.join(ROOT, "tests", "golden", "oracle_runs.json")))
    rows = []
    for c in ("C1", "C2", "C3", "C4a", "C4b", "C5"):
        p = os.path.join(d, f"bench_{c}.jsonl")
        if not os.path.exists(p):
            continue
        b = json.loads(open(p).readline())
        g = gold.get(c, {})
        ot = os.path.join(ROOT, "profiles", "r02", f"r2d_oracle_timing_{c}.json")
        ots = json.load(open(ot)) if os.path.exists(ot) else {}
        nnz = b["config"]["nnz"]
        sw1 = nnz / (b["sweep1_ms"] / 1e3)
        med = b.get("level0_sweep_median_edges_per_s")
        qa = g.get("a", {}).get("q")
        frac = b["roofline"]["frac"]
        def r(x):
            return f"{x / 1e9:.2f} G" if x >= 1e8 else f"{x / 1e6:.2f} M"
        rows.append("| {} | 1 | {} | {} | {} | {} | {:.4f} s ({:.1f} ms opt / {:.1f} ms agg, agg {:.0%}) | {:.6f} | {} | {} | yes (labels sha256 per sweep / run) | {} | {} |".format(
            NAMES[c], r(sw1), r(med) if med else "—",
            "n/a" if c == "C1" else f"{100 * frac:.1f}%",
            f"{r(b['phase1_teps_2E'])} (2\\|E\\|) / {r(b['phase1_teps_E'])} (\\|E\\|)" if b.get("phase1_teps_2E") else "—",
            b["ms_per_step"] / 1e3, b["t_opt_ms"], b["t_agg_ms"], b["agg_share"] or 0, b["q_final"],
            f"{qa:.6f}" if qa is not None else "—", f"{abs(qa - b['q_final']):.4f}" if qa is not None else "—",
            f"{ots['sweep1_s']:.2f}" if "sweep1_s" in ots else (f"{g['level0_sweeps_b'][0]['oracle_s']:.2f} (build box)" if g.get('level0_sweeps_b') else "—"),
            f"{g['a']['oracle_s']:.1f} (build box)" if g.get("a") else "—"))
    print("\n".join(rows))


if __name__ == "__main__":
    main()
