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
