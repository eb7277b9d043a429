"""Quality study (oracle only): which in-paper parameter choices close the gap between
bucket-synchronous (b) and sequential (a) Louvain on R-MAT?  SURVEY 7 hard part 1."""
import json, os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import graphgen, oracle
scale = int(sys.argv[1]) if len(sys.argv) > 1 else 20
g = graphgen.rmat(scale, seed=1)
qa = oracle.louvain(g, oracle.params(mode=oracle.SEQ)).q
rows = []
for th in (2, 3, 4, 6):
    for rule in (1, 2, 0):
        t = time.time()
        r = oracle.louvain(g, oracle.params(th_bin_exp=th, singleton_rule=rule))
        rows.append({"th_bin_exp": th, "singleton_rule": rule, "q_b": r.q, "gap": qa - r.q, "levels": r.levels,
                     "sweeps": r.sweeps, "s": time.time() - t})
        print(json.dumps(rows[-1]), flush=True)
print(json.dumps({"scale": scale, "q_a": qa}))
