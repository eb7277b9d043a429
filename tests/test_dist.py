"""Sharded sweep orchestration (paper_conf_ipps_naimmht17_b200/dist.py) on CPU:
world_size 1, 2 and 3 over gloo, each rank driving an oracle-backed engine (test
infrastructure).  The sharded run must reproduce the single-process oracle (b) run
exactly -- labels, levels, per-level sweeps and the exact modularity numerators --
because every bucket decides on one snapshot and commits are order-independent."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import graphgen
import oracle
from paper_conf_ipps_naimmht17_b200.dist import edge_balanced_ranges, run_sharded


class OracleShard:
    """Engine protocol of dist.run_sharded backed by the plain-C oracle (CPU)."""

    def __init__(self, g):
        self.g = g
        self.n, self.nnz = g.n, g.nnz
        self.st = oracle.State(g)
        self.W = self.st.W
        self.k = np.array([g.weights()[g.rowptr[i]:g.rowptr[i + 1]].sum() for i in range(g.n)], dtype=np.int64)
        self.deg = np.diff(g.rowptr)
        self.own = (0, g.n)
        self.log = []
        self.device = "cpu"

    def rowptr(self):
        return self.g.rowptr

    def set_owned_range(self, lo, hi):
        self.own = (lo, hi)

    def begin_sweep(self):
        self.log = []

    def _bucket(self, p, b):
        d = self.deg
        lo_b = 0 if b == 1 else p.deg_bounds[b - 2]
        hi_b = p.deg_bounds[b - 1] if b <= 6 else np.iinfo(np.int64).max
        sel = (d > lo_b) & (d <= hi_b)
        sel[: self.own[0]] = False
        sel[self.own[1]:] = False
        return np.flatnonzero(sel)

    def decide_bucket(self, p, b):
        verts = self._bucket(p, b)
        if len(verts) == 0:
            return torch.zeros((0, 2), dtype=torch.int32)
        t = oracle.decide_batch(self.g, self.st.C, self.st.a, self.st.size, self.W, verts, p.singleton_rule)
        mv = t != self.st.C[verts]
        return torch.from_numpy(np.stack([verts[mv], t[mv]], axis=1).astype(np.int32))

    def commit_moves(self, moves):
        for v, t in moves.numpy().tolist():
            old = int(self.st.C[v])
            self.st.a[old] -= self.k[v]
            self.st.size[old] -= 1
            self.st.a[t] += self.k[v]
            self.st.size[t] += 1
            self.st.C[v] = t
            self.log.append((v, old, t))

    def revert_sweep(self):
        for v, old, t in reversed(self.log):
            self.st.a[t] -= self.k[v]
            self.st.size[t] -= 1
            self.st.a[old] += self.k[v]
            self.st.size[old] += 1
            self.st.C[v] = old
        self.log = []

    def modularity_owned(self):
        lo, hi = self.own
        C = self.st.C
        L = 0
        w = self.g.weights()
        for i in range(lo, hi):
            for e in range(self.g.rowptr[i], self.g.rowptr[i + 1]):
                if C[self.g.col[e]] == C[i]:
                    L += int(w[e])
        S = int(np.sum(self.st.a.astype(object) ** 2))
        return L, S, self.W

    def aggregate(self):
        g2, mp = oracle.contract(self.g, self.st.C)
        return OracleShard(g2), mp

    def labels(self):
        return self.st.C.copy()

    def new_identity(self, n0):
        return np.arange(n0, dtype=np.int32)

    def compose(self, lab, mp):
        return np.asarray(mp)[lab]


GRAPHS = {
    "karate": lambda: graphgen.karate(),
    "rmat9": lambda: graphgen.rmat(9, seed=4),
    "weighted": lambda: graphgen.random_weighted(60, 0.12, 9, wmax=4, loops=True),
    "lfr": lambda: graphgen.lfr(600, kmin=4, kmax=40, smin=10, smax=80, seed=2),
}


def _check_against_oracle(name, lab, st, mode=0):
    g = GRAPHS[name]()
    r = oracle.louvain(g, oracle.params(mode=mode))
    assert st["levels"] == r.levels
    assert st["sweeps_per_level"] == r.sweeps_per_level
    assert st["num_start"] == r.num_start and st["num_end"] == r.num_end
    assert np.array_equal(np.asarray(lab), r.labels)
    assert (st["L"], st["S"]) == (r.L, r.S)


def test_edge_balanced_ranges():
    rowptr = np.array([0, 10, 10, 11, 30, 31, 40], dtype=np.int64)
    rs = edge_balanced_ranges(rowptr, 3)
    assert rs[0][0] == 0 and rs[-1][1] == 6
    assert all(a[1] == b[0] for a, b in zip(rs, rs[1:]))
    assert edge_balanced_ranges(rowptr, 1) == [(0, 6)]
    # more ranks than vertices: empty ranges are allowed, still a partition
    rs = edge_balanced_ranges(np.array([0, 2, 4], dtype=np.int64), 4)
    assert rs[0][0] == 0 and rs[-1][1] == 2 and all(a[1] == b[0] for a, b in zip(rs, rs[1:]))


@pytest.mark.parametrize("name", list(GRAPHS))
def test_world1_matches_oracle(name):
    lab, st = run_sharded(OracleShard(GRAPHS[name]()), oracle.params())
    _check_against_oracle(name, lab, st)


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _worker(rank, world, port, names, mode, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        out = {}
        for name in names:
            lab, st = run_sharded(OracleShard(GRAPHS[name]()), oracle.params(mode=mode))
            out[name] = (np.asarray(lab).tolist(), st)
        q.put((rank, out))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
@pytest.mark.parametrize("mode", [0, 1])
def test_gloo_sharded_matches_oracle(world, mode):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    names = list(GRAPHS)
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, names, mode, q)) for r in range(world)]
    for pr in procs:
        pr.start()
    results = {}
    for _ in range(world):
        rank, out = q.get(timeout=300)
        results[rank] = out
    for pr in procs:
        pr.join(timeout=60)
        assert pr.exitcode == 0
    for name in names:
        lab0, st0 = results[0][name]
        for r in range(1, world):  # replicas identical on every rank
            assert results[r][name][0] == lab0 and results[r][name][1] == st0
        _check_against_oracle(name, lab0, st0, mode=mode)
