"""Pins of the oracle's multilevel driver and contraction:
* brute force over all partitions (n <= 9): no Louvain result exceeds Q_opt;
* contraction == P^T A P (scipy sparse; Alg. 3, R17/R18), W preserved,
  Q(singletons of G') == Q(C on G) exactly;
* karate (C1): oracle (a) reaches the north star's Q ~ 0.4188; no result exceeds
  the literature optimum 0.4197896 (Brandes et al., PAPER.md ref [2]);
* golden regression tests/golden/karate_trace.json (SURVEY 8(c) [proto] trace).
"""
import json
import os
from fractions import Fraction

import numpy as np
import pytest

import graphgen
import oracle
from refq import dense_adj, q_dense, q_dense_float_many, set_partitions

GOLD = os.path.join(os.path.dirname(__file__), "golden")
KARATE_OPT = 0.4197896  # Brandes et al. (PAPER.md [2]); upper bound for any partition


def bruteforce_opt(g) -> float:
    A = dense_adj(g)
    parts = np.array(list(set_partitions(g.n)), dtype=np.int32)
    return float(q_dense_float_many(A, parts).max())


def test_bell_numbers():
    assert [sum(1 for _ in set_partitions(n)) for n in range(1, 8)] == [1, 2, 5, 15, 52, 203, 877]


@pytest.mark.parametrize("seed", range(8))
def test_never_above_bruteforce_optimum(seed):
    rng = np.random.default_rng(seed)
    n = int(rng.integers(4, 9))
    g = graphgen.random_weighted(n, 0.45, seed + 50, wmax=3, loops=bool(seed % 2))
    if g.nnz == 0:
        pytest.skip("empty")
    qopt = bruteforce_opt(g)
    A = dense_adj(g)
    for mode in (oracle.BIN_SYNC, oracle.RELAXED, oracle.SEQ):
        r = oracle.louvain(g, oracle.params(mode=mode))
        q_labels = float(q_dense(A, r.labels))
        assert abs(q_labels - r.q) < 1e-12  # reported Q is Q of the returned labels
        assert r.q <= qopt + 1e-12
        assert r.q >= float(q_dense(A, np.arange(n))) - 1e-12  # never below the start (R15)


@pytest.mark.parametrize("seed", range(10))
def test_contract_is_PtAP_and_preserves_Q(seed):
    sp = pytest.importorskip("scipy.sparse")
    rng = np.random.default_rng(seed)
    n = int(rng.integers(3, 40))
    g = graphgen.random_weighted(n, 0.3, seed + 7, wmax=6, loops=True)
    if g.nnz == 0:
        pytest.skip("empty")
    C = rng.integers(0, max(1, n // 3), size=n).astype(np.int32)
    g2, mp = oracle.contract(g, C)
    A = sp.csr_matrix((g.weights().astype(np.int64), g.col, g.rowptr), shape=(n, n))
    labels = np.unique(C)
    P = sp.csr_matrix((np.ones(n, dtype=np.int64), (np.arange(n), np.searchsorted(labels, C))),
                      shape=(n, len(labels)))
    B = (P.T @ A @ P).toarray()
    A2 = sp.csr_matrix((g2.weights().astype(np.int64), g2.col, g2.rowptr), shape=(g2.n, g2.n)).toarray()
    assert g2.n == len(labels)
    assert np.array_equal(A2, B)
    assert mp.tolist() == np.searchsorted(labels, C).tolist()
    for r in range(g2.n):  # rows sorted by column, no duplicates
        row = g2.col[g2.rowptr[r]:g2.rowptr[r + 1]]
        assert np.all(np.diff(row) > 0)
    L, S, W = oracle.modularity(g, C)
    L2, S2, W2 = oracle.modularity(g2, np.arange(g2.n))
    assert W2 == W and L2 * W2 - S2 == L * W - S


def test_karate_sequential_matches_north_star(karate):
    r = oracle.louvain(karate, oracle.params(mode=oracle.SEQ))
    assert abs(r.q - 0.4188) < 5e-5  # BASELINE.json north star: "Q~0.4188 for Louvain"
    assert r.q <= KARATE_OPT


def test_karate_sync_bounded_by_optimum(karate):
    r = oracle.louvain(karate)
    assert r.q <= KARATE_OPT + 1e-7
    assert abs(r.q - oracle.louvain(karate, oracle.params(mode=oracle.SEQ)).q) <= 0.005  # north-star bar


def test_karate_golden_trace(karate):
    with open(os.path.join(GOLD, "karate_trace.json")) as f:
        gold = json.load(f)
    st = oracle.State(karate)
    p = oracle.params()
    for sw in gold["level0_sweeps"]:
        moved = st.sweep(p)
        L, S, W = st.qnum()
        assert moved == sw["moved"]
        assert abs((L * W - S) / W / W - sw["q"]) < 5e-7
        if "labels" in sw:
            assert st.C.tolist() == sw["labels"]
    r = oracle.louvain(karate)
    assert r.levels == gold["levels"]
    assert r.sweeps_per_level == gold["sweeps_per_level"]
    assert r.n == gold["n_per_level"] and r.nnz == gold["nnz_per_level"]
    assert abs(r.q - gold["q_final"]) < 5e-9
    rs = oracle.louvain(karate, oracle.params(mode=oracle.SEQ))
    assert abs(rs.q - gold["q_seq"]) < 5e-7
    assert rs.sweeps_per_level == gold["seq_sweeps_per_level"]


def test_revert_keeps_phase_above_start():
    # R15: random small graphs; every level's end numerator >= its start numerator.
    for seed in range(30):
        g = graphgen.random_weighted(7, 0.5, 300 + seed, wmax=3, loops=False)
        if g.nnz == 0:
            continue
        r = oracle.louvain(g)
        for s, e in zip(r.num_start, r.num_end):
            assert e >= s


def test_threshold_schedule_size_limit():
    # n > limit uses t_bin.  With limit 0 the level-0 phase stops after the
    # first sweep whose gain < 1e-2; it can never run more sweeps than with t_final.
    g = graphgen.rmat(11, seed=5)
    r_bin = oracle.louvain(g, oracle.params(size_limit=0))
    r_fin = oracle.louvain(g)  # n < 100000 -> t_final everywhere
    assert r_bin.sweeps_per_level[0] <= r_fin.sweeps_per_level[0]
    L, S, W = oracle.modularity(g, r_bin.labels)
    assert abs((L * W - S) / W / W - r_bin.q) < 1e-12


def test_empty_and_degenerate():
    g = graphgen.from_edges(3, [], [], compact=False)  # no edges: W = 0
    r = oracle.louvain(g)
    assert r.levels == 0 and r.labels.tolist() == [0, 1, 2]
    g1 = graphgen.weighted_csr(1, [0], [0], [3])  # one vertex with a self-loop
    r1 = oracle.louvain(g1)
    assert r1.q == 0.0 and r1.labels.tolist() == [0]


def test_relaxed_is_one_bucket(karate):
    # RELAXED = all vertices in a single bucket; equivalent to deg_bounds so
    # large that every vertex falls in bucket 1.
    s1 = oracle.State(karate)
    s1.sweep(oracle.params(mode=oracle.RELAXED))
    s2 = oracle.State(karate)
    s2.sweep(oracle.params(deg_bounds=[10**9] * 6))
    assert s1.C.tolist() == s2.C.tolist()


def _star5():
    # K_{1,5}: hub 0, leaves 1..5, unit weights; W = 2m = 10, k = (5, 1, 1, 1, 1, 1)
    return graphgen.from_edges(6, [0, 0, 0, 0, 0], [1, 2, 3, 4, 5], compact=False)


def test_relaxed_worked_star():
    """RELAXED decides every vertex on ONE snapshot, BIN_SYNC commits bucket 1
    (the leaves, deg 1) before bucket 2 (the hub, deg 5) decides (Alg. 1 l.4-11).
    Hand computation with the singleton rule off (rule 0), from singletons:
      leaf i: one candidate, the hub: s = W*1 - k_i*a_0 = 10 - 5 = 5 > s_stay = 0 -> moves to 0;
      hub, RELAXED (all singletons): every leaf c has s = 10*1 - 5*1 = 5, tie -> lowest label 1,
        s_stay = 10*0 - 5*(5 - 5) = 0 -> moves to 1;
      hub, BIN_SYNC (leaves already in 0): its only label is its own -> stays.
    RELAXED: C = [1,0,0,0,0,0], L = 0, a = {0: 5, 1: 5}, S = 50, Q = (0*10 - 50)/100 = -1/2.
    BIN_SYNC: C = [0]*6, L = 10, S = 100, Q = 0.  With the veto rule (1) the RELAXED hub's
    best (label 1 > own 0, both singletons) is vetoed: C = [0]*6."""
    g = _star5()
    st = oracle.State(g)
    assert st.sweep(oracle.params(mode=oracle.RELAXED, singleton_rule=0)) == 6
    assert st.C.tolist() == [1, 0, 0, 0, 0, 0]
    assert st.qnum() == (0, 50, 10)
    st = oracle.State(g)
    assert st.sweep(oracle.params(mode=oracle.BIN_SYNC, singleton_rule=0)) == 5
    assert st.C.tolist() == [0] * 6 and st.qnum() == (10, 100, 10)
    st = oracle.State(g)
    assert st.sweep(oracle.params(mode=oracle.RELAXED, singleton_rule=1)) == 5
    assert st.C.tolist() == [0] * 6
    # whole run, RELAXED rule 0: the sweep lowers Q from -30/100 (singletons: S = 25 + 5)
    # to -50/100, so it is reverted (R15) and nothing moved: labels stay singletons
    r = oracle.louvain(g, oracle.params(mode=oracle.RELAXED, singleton_rule=0))
    assert r.labels.tolist() == [0, 1, 2, 3, 4, 5] and (r.L, r.S, r.W) == (0, 30, 10)
    assert r.levels == 1 and r.sweeps_per_level == [1]


def test_adaptive_sequential_worked_path():
    """Sequential Louvain (R23) and its adaptive variant (the n-dependent
    threshold theta_bin while n > size_limit) on the path 0-1-2-3 (W = 6, k = (1, 2, 2, 1)).
    Hand computation, ascending ids, immediate updates, no singleton rule:
      sweep 1: v0 -> 1 (s = 6 - 1*2 = 4 > 0); v1 stays (s_stay = 6*1 - 2*(3-2) = 4 > s_2 = 6 - 2*2 = 2);
               v2 -> 3 (s_3 = 6 - 2*1 = 4 > s_1 = 6 - 2*3 = 0 = s_stay); v3 stays.
               C = [1,1,3,3], numerator L*W - S = 4*6 - 18 = 6 (start: 0 - 10 = -10).
      sweep 2: nothing moves -> phase ends after 2 sweeps (theta_final = 1e-6).
      level 1: two vertices, self-loops 2, edge weight 1, k = 3: s = 6*1 - 3*3 = -3 < 0, no move.
    Adaptive with size_limit = 2 and theta_bin = 10^0: level 0 (n = 4 > 2) stops after sweep 1
    because (6 - (-10)) * 10^0 < W^2 = 36; the labels are the same."""
    g = graphgen.from_edges(4, [0, 1, 2], [1, 2, 3], compact=False)
    st = oracle.State(g)
    assert st.sweep(oracle.params(mode=oracle.SEQ)) == 2
    assert st.C.tolist() == [1, 1, 3, 3] and st.qnum() == (4, 18, 6)
    r = oracle.louvain(g, oracle.params(mode=oracle.SEQ))
    assert r.sweeps_per_level == [2, 1] and r.labels.tolist() == [0, 0, 1, 1]
    assert (r.L * r.W - r.S, r.num_start) == (6, [-10, 6])
    ra = oracle.louvain(g, oracle.params(mode=oracle.SEQ_ADAPTIVE, size_limit=2, th_bin_exp=0))
    assert ra.sweeps_per_level == [1, 1] and ra.labels.tolist() == [0, 0, 1, 1]
    # n <= size_limit at every level: adaptive == sequential exactly
    for gg in (g, graphgen.karate(), graphgen.rmat(9, seed=4)):
        a = oracle.louvain(gg, oracle.params(mode=oracle.SEQ))
        b = oracle.louvain(gg, oracle.params(mode=oracle.SEQ_ADAPTIVE))
        assert a.labels.tolist() == b.labels.tolist() and a.sweeps_per_level == b.sweeps_per_level


def test_adaptive_theta_one_sweep_per_large_level():
    # theta_bin = 10^0 and size_limit = 0: every level runs exactly one sweep (a Q gain is < 1)
    g = graphgen.rmat(10, seed=3)
    r = oracle.louvain(g, oracle.params(mode=oracle.SEQ_ADAPTIVE, size_limit=0, th_bin_exp=0))
    assert all(s == 1 for s in r.sweeps_per_level)
    L, S, W = oracle.modularity(g, r.labels)
    assert (L, S) == (r.L, r.S)


def test_sweep_D_count():
    """D of the byte model: distinct (i, c != C(i)) pairs evaluated by a sweep.
    Closed form on a simple graph from singletons under RELAXED (one snapshot, every neighbour
    its own label): D = nnz - (number of self-loop entries) = nnz.  Under BIN_SYNC later buckets
    see merged labels, so D <= nnz; the counted sweep moves exactly like the plain one."""
    for g in (graphgen.karate(), graphgen.rmat(10, seed=3), graphgen.lfr(2000, kmin=4, kmax=60, smin=20,
                                                                              smax=200, seed=4)):
        st = oracle.State(g)
        moved, D = st.sweep_counted(oracle.params(mode=oracle.RELAXED))
        assert D == g.nnz
        s1, s2 = oracle.State(g), oracle.State(g)
        m1, D1 = s1.sweep_counted(oracle.params())
        m2 = s2.sweep(oracle.params())
        assert m1 == m2 and s1.C.tolist() == s2.C.tolist() and D1 <= g.nnz
    # a weighted graph with self-loops: the loop is not a candidate (R3)
    g = graphgen.weighted_csr(3, [0, 0, 1], [0, 1, 2], [5, 1, 2])
    _, D = oracle.State(g).sweep_counted(oracle.params(mode=oracle.RELAXED))
    assert D == g.nnz - 1
