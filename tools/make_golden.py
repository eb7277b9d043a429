"""Write tests/golden/oracle_runs.json: full-run results of the ORACLE ONLY (oracle
(b) bucket-synchronous and oracle (a) sequential Louvain) on the synthetic configs,
built with the host generators.  The GPU tests compare the CUDA path against these
stored values (exact numerators, levels, sweeps per level, sha256 of the labels)
and check the north-star quality bar |Q_b - Q_a| <= 0.005.

    python tools/make_golden.py [config ...]      (CPU only; minutes for the big ones)
"""
import hashlib
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

import graphgen  # noqa: E402
import oracle  # noqa: E402

OUT = os.path.join(ROOT, "tests", "golden", "oracle_runs.json")

CONFIGS = {
    # name: (builder, description)
    "C1": (lambda: graphgen.karate(), "Zachary karate club"),
    "C2-small": (lambda: graphgen.lfr(20_000, seed=1), "LFR-style n=20000 (C2 recipe scaled)"),
    "C3-small": (lambda: graphgen.rmat(16, seed=1), "R-MAT scale 16 (C3/C5 recipe scaled)"),
    "C4a-small": (lambda: graphgen.mesh3d(40, True), "3-D mesh 40^3, Morton ids (C4a recipe scaled)"),
    "C4b-small": (lambda: graphgen.rgg(200_000, seed=1), "RGG n=200000 (C4b recipe scaled)"),
    "C2": (lambda: graphgen.lfr(1_000_000, seed=1), "LFR-style n=1e6 (C2)"),
    "C3-s20": (lambda: graphgen.rmat(20, seed=1), "R-MAT scale 20"),
    "C3": (lambda: graphgen.rmat(24, seed=1), "R-MAT scale 24 (C3)"),
    "C4a": (lambda: graphgen.mesh3d(368, True), "3-D 7-point mesh 368^3, Morton ids (C4a)"),
    "C4b": (lambda: graphgen.rgg(50_000_000, seed=1), "RGG n=5e7, r = 0.55 sqrt(ln n / n) (C4b)"),
    "C5": (lambda: graphgen.rmat(27, seed=1), "R-MAT scale 27 (C5, the bench workload)"),
}


def labels_sha(lab) -> str:
    return hashlib.sha256(np.ascontiguousarray(lab, dtype=np.int32).tobytes()).hexdigest()


def run(name, sweeps_only=False):
    build, desc = CONFIGS[name]
    t0 = time.time()
    g = build()
    tg = time.time() - t0
    res = {"desc": desc, "n": g.n, "nnz": g.nnz, "gen_s": tg}
    # level-0 sweeps 1 and 2 of oracle (b) from singletons (one louvain_sweep each):
    # full-label sha256, moved count and exact Eq. (1) parts after each sweep
    st = oracle.State(g)
    p = oracle.params()
    sw = []
    for s in range(2):
        t0 = time.time()
        moved, D = st.sweep_counted(p)  # D: distinct (vertex, candidate label) pairs (byte model)
        L, S, W = st.qnum()
        sw.append({"moved": moved, "D": D, "L": L, "S": S, "W": W, "labels_sha256": labels_sha(st.C),
                   "oracle_s": time.time() - t0})
    res["level0_sweeps_b"] = sw
    del st
    if sweeps_only:
        return res
    for tag, mode in (("b", oracle.BIN_SYNC), ("a", oracle.SEQ), ("a_adaptive", oracle.SEQ_ADAPTIVE)):
        t0 = time.time()
        r = oracle.louvain(g, oracle.params(mode=mode))
        res[tag] = {"q": r.q, "L": r.L, "S": r.S, "W": r.W, "levels": r.levels,
                    "sweeps_per_level": r.sweeps_per_level, "n_per_level": r.n, "nnz_per_level": r.nnz,
                    "num_start": r.num_start, "num_end": r.num_end, "labels_sha256": labels_sha(r.labels),
                    "communities": int(len(np.unique(r.labels))), "oracle_s": time.time() - t0}
    if g.labels is not None:  # planted partition: Q of the ground truth
        L, S, W = oracle.modularity(g, g.labels)
        res["q_ground_truth"] = (L * W - S) / W / W
    res["gap_a_minus_b"] = res["a"]["q"] - res["b"]["q"]
    res["gap_a_adaptive_minus_b"] = res["a_adaptive"]["q"] - res["b"]["q"]
    return res


def main():
    args = [a for a in sys.argv[1:] if not a.startswith("--")]
    sweeps_only = "--sweeps-only" in sys.argv  # level-0 sweeps 1-2 only (merged into the config's record)
    names = args or list(CONFIGS)
    data = {}
    if os.path.exists(OUT):
        with open(OUT) as f:
            data = json.load(f)
    data["_source"] = ("tools/make_golden.py: oracle/ only (plain C, single thread), host graph builders of "
                       "graphgen/; see DESIGN.md 'Input recipe'")
    for name in names:
        print(f"[{time.strftime('%X')}] {name} ...", flush=True)
        if sweeps_only:
            cur = json.load(open(OUT)) if os.path.exists(OUT) else {}
            rec = cur.get(name, {})
            rec["level0_sweeps_b"] = run(name, True)["level0_sweeps_b"]
            cur[name] = rec
            with open(OUT, "w") as f:
                json.dump(cur, f, indent=1, sort_keys=True)
            print(f"   {name}: level-0 sweeps {rec['level0_sweeps_b']}", flush=True)
            continue
        data[name] = run(name)
        print(f"   b: Q={data[name]['b']['q']:.6f} levels={data[name]['b']['levels']}  "
              f"a: Q={data[name]['a']['q']:.6f}  gap={data[name]['gap_a_minus_b']:+.5f}  "
              f"a_adaptive: Q={data[name]['a_adaptive']['q']:.6f} "
              f"({data[name]['b']['oracle_s']:.0f}s + {data[name]['a']['oracle_s']:.0f}s"
              f" + {data[name]['a_adaptive']['oracle_s']:.0f}s)", flush=True)
        cur = {}
        if os.path.exists(OUT):  # merge: several configs may be generated by concurrent processes
            with open(OUT) as f:
                cur = json.load(f)
        cur["_source"] = data["_source"]
        cur[name] = data[name]
        with open(OUT, "w") as f:
            json.dump(cur, f, indent=1, sort_keys=True)


if __name__ == "__main__":
    main()
