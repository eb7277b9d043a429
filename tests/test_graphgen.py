"""Input generators (SURVEY 8(d) recipes): structural checks
on the host builders.  Host == device bit-identity is checked in test_gpu_parity.py."""
import numpy as np
import pytest

import graphgen

KARATE_DEG = [16, 9, 10, 6, 3, 4, 4, 4, 5, 2, 3, 1, 2, 5, 2, 2, 2, 2, 2, 3, 2, 2, 2, 5, 3, 3, 2, 4, 3, 4, 4, 6, 12, 17]


def canonical(g):
    """symmetric, sorted rows, no self-loops, no duplicates, no isolated vertices"""
    deg = np.diff(g.rowptr)
    src = np.repeat(np.arange(g.n), deg)
    assert np.all(src != g.col), "self-loop"
    for i in range(min(g.n, 5000)):
        row = g.col[g.rowptr[i]:g.rowptr[i + 1]]
        assert np.all(np.diff(row) > 0), "unsorted or duplicate"
    fwd = set(zip(src.tolist(), g.col.tolist()))
    assert all((v, u) in fwd for (u, v) in fwd), "asymmetric"
    return deg


def test_karate_appendix_b(karate):
    assert karate.n == 34 and karate.nnz == 156
    assert np.diff(karate.rowptr).tolist() == KARATE_DEG
    assert int(np.sum(np.array(KARATE_DEG) ** 2)) == 1212
    canonical(karate)


def test_from_edges_dedup_and_loops():
    g = graphgen.from_edges(5, [0, 1, 0, 2, 3], [1, 0, 0, 3, 2])
    # (0,1) twice, loop (0,0) dropped, (2,3) twice; vertex 4 isolated -> compacted
    assert g.n == 4 and g.nnz == 4
    canonical(g)


@pytest.mark.parametrize("scale", [8, 12])
def test_rmat_canonical_and_deterministic(scale):
    g = graphgen.rmat(scale, seed=1)
    deg = canonical(g)
    assert deg.min() >= 1
    g2 = graphgen.rmat(scale, seed=1)
    assert np.array_equal(g.rowptr, g2.rowptr) and np.array_equal(g.col, g2.col)
    g3 = graphgen.rmat(scale, seed=2)
    assert not (g3.nnz == g.nnz and np.array_equal(g3.col, g.col))
    # skew: unscrambled R-MAT puts the hub at a low id
    assert int(np.argmax(deg)) < g.n // 16


def test_rmat_no_compact_keeps_vertex_space():
    g = graphgen.rmat(8, compact=False)
    assert g.n == 256


def test_mesh_row_major_counts():
    L = 5
    g = graphgen.mesh3d(L, morton=False)
    deg = canonical(g)
    assert g.n == L ** 3 and g.nnz == 6 * L ** 3 - 6 * L * L
    assert sorted(set(deg.tolist())) == [3, 4, 5, 6]
    assert deg[0] == 3  # corner


def _morton(x, y, z, bits):
    c = 0
    for b in range(bits):
        c |= ((x >> b) & 1) << (3 * b) | ((y >> b) & 1) << (3 * b + 1) | ((z >> b) & 1) << (3 * b + 2)
    return c


@pytest.mark.parametrize("L", [4, 6])
def test_mesh_morton_is_relabelled_mesh(L):
    gm = graphgen.mesh3d(L, morton=True)
    gr = graphgen.mesh3d(L, morton=False)
    bits = max(1, int(np.ceil(np.log2(L))))
    coords = [(x, y, z) for z in range(L) for y in range(L) for x in range(L)]  # row-major index order
    codes = np.array([_morton(x, y, z, bits) for (x, y, z) in coords])
    rank = np.empty(len(codes), dtype=np.int64)
    rank[np.argsort(codes, kind="stable")] = np.arange(len(codes))  # id = rank of Morton code
    er = set()
    for i in range(gr.n):
        for e in range(gr.rowptr[i], gr.rowptr[i + 1]):
            er.add((int(rank[i]), int(rank[gr.col[e]])))
    em = set()
    for i in range(gm.n):
        for e in range(gm.rowptr[i], gm.rowptr[i + 1]):
            em.add((i, int(gm.col[e])))
    assert er == em


def test_rgg_canonical_and_degree():
    n = 20000
    g = graphgen.rgg(n, seed=3)
    canonical(g)
    r = 0.55 * np.sqrt(np.log(n) / n)
    mean_deg = g.nnz / n
    expect = np.pi * r * r * n  # boundary effects lower it slightly
    assert 0.85 * expect < mean_deg < 1.02 * expect


def test_lfr_small():
    n = 5000
    g = graphgen.lfr(n, kmin=8, kmax=100, smin=20, smax=500, mu=0.3, seed=4)
    canonical(g)
    assert g.labels is not None and len(g.labels) == g.n
    src = np.repeat(np.arange(g.n), np.diff(g.rowptr))
    intra = np.mean(g.labels[src] == g.labels[g.col])
    assert 0.6 < intra < 0.8  # ~ 1 - mu after dedup
