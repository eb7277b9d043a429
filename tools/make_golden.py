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


def run(name):
    build, desc = CONFIGS[name]
    t0 = time.time()
    g = build()
    tg = time.time() - t0
    res = {"desc": desc, "n": g.n, "nnz": g.nnz, "gen_s": tg}
    for tag, mode in (("b", oracle.BIN_SYNC), ("a", oracle.SEQ)):
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
    return res


def main():
    names = sys.argv[1:] or list(CONFIGS)
    data = {}
    if os.path.exists(OUT):
        with open(OUT) as f:
            data = json.load(f)
    data["_source"] = ("tools/make_golden.py: oracle/ only (plain C, single thread), host graph builders of "
                       "graphgen/; see DESIGN.md 'Input recipe'")
    for name in names:
        print(f"[{time.strftime('%X')}] {name} ...", flush=True)
        data[name] = run(name)
        print(f"   b: Q={data[name]['b']['q']:.6f} levels={data[name]['b']['levels']}  "
              f"a: Q={data[name]['a']['q']:.6f}  gap={data[name]['gap_a_minus_b']:+.5f}  "
              f"({data[name]['b']['oracle_s']:.0f}s + {data[name]['a']['oracle_s']:.0f}s)", flush=True)
        with open(OUT, "w") as f:
            json.dump(data, f, indent=1, sort_keys=True)


if __name__ == "__main__":
    main()
