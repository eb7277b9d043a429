"""The graph-file loader of the input module (graphgen/csrc/graph_io.cpp): Matrix Market,
edge lists and the binary .csrbin container, to the R1 CSR the method reads (CSR
with both directions of every edge; self-loop stored once)."""
import os

import numpy as np
import pytest

import graphgen

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def same(a, b):
    return (a.n == b.n and np.array_equal(a.rowptr, b.rowptr) and np.array_equal(a.col, b.col)
            and ((a.w is None and b.w is None) or np.array_equal(a.weights(), b.weights())))


def test_karate_mtx_fixture_equals_generator():
    g = graphgen.load(os.path.join(GOLD, "karate.mtx"))
    k = graphgen.karate()
    assert same(g, k) and g.w is None
    deg = np.diff(g.rowptr)
    assert deg.sum() == 156 and int((deg.astype(np.int64) ** 2).sum()) == 1212


def test_csrbin_round_trip(tmp_path):
    for g in (graphgen.karate(), graphgen.random_weighted(40, 0.2, 3, wmax=9, loops=True), graphgen.rmat(10, seed=2)):
        p = str(tmp_path / "g.csrbin")
        graphgen.save_csrbin(g, p)
        h = graphgen.load(p)
        assert same(g, h)


def test_edge_list_weighted_with_loops_and_repeats(tmp_path):
    p = tmp_path / "e.txt"
    p.write_text("# comment\n0 1 2\n1 2 3\n% another\n2 2 5\n1 0 1\n\n3 1 4\n")
    g = graphgen.load(str(p))
    # {0,1}: 2 + 1 (repeat, reversed), {1,2}: 3, loop {2}: 5 once, {1,3}: 4
    assert g.n == 4
    rows = {u: dict(zip(g.col[g.rowptr[u]:g.rowptr[u + 1]].tolist(), g.w[g.rowptr[u]:g.rowptr[u + 1]].tolist()))
            for u in range(g.n)}
    assert rows == {0: {1: 3}, 1: {0: 3, 2: 3, 3: 4}, 2: {1: 3, 2: 5}, 3: {1: 4}}
    assert int(g.weights().sum()) == 2 * (3 + 3 + 4) + 5  # W = 2m, loop once (R1)


def test_edge_list_unweighted_is_simple_and_one_based_guess(tmp_path):
    p = tmp_path / "e.el"
    p.write_text("1 2\n2 1\n2 3\n1 2\n")  # no id 0 -> 1-based
    g = graphgen.load(str(p))
    assert g.w is None and g.n == 3
    assert g.rowptr.tolist() == [0, 1, 3, 4] and g.col.tolist() == [1, 0, 2, 1]
    g0 = graphgen.load(str(p), one_based=False)  # forced 0-based: vertex 0 isolated
    assert g0.n == 4 and g0.rowptr.tolist()[:2] == [0, 0]
    gc = graphgen.load(str(p), one_based=False, compact=True)  # R21: isolated vertices dropped
    assert same(gc, g)


def test_mtx_integer_general(tmp_path):
    p = tmp_path / "w.mtx"
    p.write_text("%%MatrixMarket matrix coordinate integer general\n%\n3 3 3\n1 2 7\n3 3 2\n2 3 1\n")
    g = graphgen.load(str(p))
    assert g.n == 3 and g.rowptr.tolist() == [0, 1, 3, 5]
    assert g.col.tolist() == [1, 0, 2, 1, 2] and g.w.tolist() == [7, 7, 1, 1, 2]


@pytest.mark.parametrize("text,msg", [
    ("%%MatrixMarket matrix array real general\n2 2\n1\n2\n3\n4\n", "coordinate"),
    ("%%MatrixMarket matrix coordinate real symmetric\n2 2 1\n2 1 0.5\n", "positive integers"),
    ("%%MatrixMarket matrix coordinate pattern symmetric\n2 3 1\n2 1\n", "square"),
    ("%%MatrixMarket matrix coordinate pattern symmetric\n2 2 2\n2 1\n", "truncated"),
    ("%%MatrixMarket matrix coordinate pattern symmetric\n2 2 1\n3 1\n", "out of range"),
])
def test_mtx_errors(tmp_path, text, msg):
    p = tmp_path / "bad.mtx"
    p.write_text(text)
    with pytest.raises(ValueError, match=msg):
        graphgen.load(str(p))


def test_csrbin_rejects_corruption(tmp_path):
    p = str(tmp_path / "g.csrbin")
    graphgen.save_csrbin(graphgen.karate(), p)
    data = bytearray(open(p, "rb").read())
    data[32 + 8 * 35 + 4 * 3] = 0xFF  # a column id beyond n
    data[32 + 8 * 35 + 4 * 3 + 3] = 0x7F
    open(p, "wb").write(bytes(data))
    with pytest.raises(ValueError, match="invalid CSR"):
        graphgen.load(p)
