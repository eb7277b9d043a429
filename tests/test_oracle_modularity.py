"""Pins of the oracle's Eq. (1) against things
other than itself: closed forms, the dense textbook double sum (tests/refq.py)
and networkx (an independent library)."""
from fractions import Fraction

import numpy as np
import pytest

import graphgen
import oracle
from refq import dense_adj, q_dense


def qfrac(g, C) -> Fraction:
    L, S, W = oracle.modularity(g, C)
    return Fraction(L * W - S, W * W)


def test_karate_singletons_closed_form(karate):
    # singleton partition: Q = sum_i A_ii/2m - sum_i k_i^2/(2m)^2; karate: 0 - 1212/156^2 = -101/2028
    assert qfrac(karate, np.arange(34)) == Fraction(-101, 2028)


def test_all_in_one_is_zero(karate):
    assert qfrac(karate, np.zeros(34, dtype=np.int32)) == 0


def _clique_edges(s, off):
    return [(off + i, off + j) for i in range(s) for j in range(i + 1, s)]


@pytest.mark.parametrize("s", [3, 4, 7])
def test_two_disjoint_cliques_half(s):
    e = _clique_edges(s, 0) + _clique_edges(s, s)
    g = graphgen.from_edges(2 * s, [a for a, _ in e], [b for _, b in e])
    C = np.array([0] * s + [1] * s, dtype=np.int32)
    assert qfrac(g, C) == Fraction(1, 2)


@pytest.mark.parametrize("r,s", [(3, 3), (5, 6), (8, 4)])
def test_ring_of_cliques_closed_form(r, s):
    e = []
    for c in range(r):
        e += _clique_edges(s, c * s)
        e.append((c * s, ((c + 1) % r) * s + 1))  # one edge to the next clique
    g = graphgen.from_edges(r * s, [a for a, _ in e], [b for _, b in e])
    C = np.repeat(np.arange(r), s).astype(np.int32)
    l = s * (s - 1) // 2
    d = s * (s - 1) + 2
    m = r * l + r
    expect = r * (Fraction(l, m) - Fraction(d, 2 * m) ** 2)
    assert qfrac(g, C) == expect
    if (r, s) == (5, 6):
        assert abs(float(expect) - 0.7375) < 1e-12  # SURVEY 8(c) pin table value


@pytest.mark.parametrize("seed", range(12))
def test_matches_dense_textbook_with_loops_and_weights(seed):
    rng = np.random.default_rng(seed)
    n = int(rng.integers(2, 14))
    g = graphgen.random_weighted(n, 0.4, seed, wmax=7, loops=True)
    if g.nnz == 0:
        pytest.skip("empty draw")
    A = dense_adj(g)
    for _ in range(5):
        C = rng.integers(0, max(1, n // 2), size=n).astype(np.int32)
        assert qfrac(g, C) == q_dense(A, C)


def test_singletons_closed_form_with_loops():
    # Q(singletons) = sum_i A_ii / 2m - sum_i k_i^2 / (2m)^2 with A_ii the stored loop weight
    g = graphgen.weighted_csr(4, [0, 1, 2, 0, 3], [0, 2, 3, 1, 3], [5, 2, 1, 3, 4])
    k = np.array([5 + 3, 3 + 2, 2 + 1, 1 + 4])
    two_m = int(k.sum())
    expect = Fraction(5 + 4, two_m) - Fraction(int((k * k).sum()), two_m * two_m)
    assert qfrac(g, np.arange(4)) == expect


@pytest.mark.parametrize("seed", range(6))
def test_matches_networkx(seed):
    nx = pytest.importorskip("networkx")
    rng = np.random.default_rng(100 + seed)
    n = 60
    g = graphgen.random_weighted(n, 0.1, seed, wmax=4, loops=False)  # networkx counts loops twice
    G = nx.Graph()
    G.add_nodes_from(range(n))
    w = g.weights()
    for i in range(n):
        for e in range(g.rowptr[i], g.rowptr[i + 1]):
            j = int(g.col[e])
            if i < j:
                G.add_edge(i, j, weight=int(w[e]))
    for _ in range(4):
        C = rng.integers(0, 7, size=n).astype(np.int32)
        comms = [set(np.flatnonzero(C == c).tolist()) for c in np.unique(C)]
        ref = nx.community.modularity(G, comms, weight="weight")
        assert abs(float(qfrac(g, C)) - ref) < 1e-12


def test_karate_networkx_unweighted(karate):
    nx = pytest.importorskip("networkx")
    G = nx.karate_club_graph()
    rng = np.random.default_rng(7)
    for _ in range(5):
        C = rng.integers(0, 4, size=34).astype(np.int32)
        comms = [set(np.flatnonzero(C == c).tolist()) for c in np.unique(C)]
        ref = nx.community.modularity(G, comms, weight=None)  # karate_club_graph carries weights 1-7: ignore
        assert abs(float(qfrac(karate, C)) - ref) < 1e-12


def test_overflow_guard():
    # W > 3,037,000,499 must be refused (R4: W^2 < 2^63)
    g = graphgen.weighted_csr(2, [0], [1], [1_600_000_000])
    with pytest.raises(OverflowError):
        oracle.modularity(g, np.arange(2))


def _delta_L(g, C0, C1):
    """The identity the GPU delta pass of Eq. (1) evaluates (DESIGN a5): only entries with a
    moved endpoint change L; from each moved row, an entry to an unmoved j counts twice (its
    mirror has the same weight and the same change), to a moved j once."""
    w = g.w if g.w is not None else np.ones(len(g.col), dtype=np.int64)
    moved = C0 != C1
    d = 0
    for i in np.flatnonzero(moved):
        for e in range(g.rowptr[i], g.rowptr[i + 1]):
            j = g.col[e]
            if j == i:
                continue
            ch = int(C1[j] == C1[i]) - int(C0[j] == C0[i])
            d += ch * int(w[e]) * (1 if moved[j] else 2)
    return d


@pytest.mark.parametrize("maker", [lambda: graphgen.karate(), lambda: graphgen.rmat(10, seed=3),
                                   lambda: graphgen.weighted_csr(60, [0, 1, 2, 3, 4, 5, 0, 7], [0, 2, 3, 3, 9, 6, 7, 8],
                                                                 [5, 1, 2, 7, 1, 3, 2, 4])])
def test_delta_identity_against_eq1(maker):
    """Pin of the delta-pass reading: L(after) - L(before) of a real sweep (oracle (b)) and of
    random relabellings equals the moved-rows sum, with L from Eq. (1) (orc_modularity)."""
    g = maker()
    rng = np.random.default_rng(0)
    st = oracle.State(g)
    for _ in range(3):
        C0 = st.C.copy()
        st.sweep(oracle.params())
        C1 = st.C.copy()
        assert oracle.modularity(g, C1)[0] - oracle.modularity(g, C0)[0] == _delta_L(g, C0, C1)
    for _ in range(3):
        C0 = rng.integers(0, max(2, g.n // 3), size=g.n).astype(np.int32)
        C1 = C0.copy()
        flip = rng.random(g.n) < 0.3
        C1[flip] = rng.integers(0, max(2, g.n // 3), size=int(flip.sum()))
        assert oracle.modularity(g, C1)[0] - oracle.modularity(g, C0)[0] == _delta_L(g, C0, C1)
