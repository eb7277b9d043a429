"""The vertex-sharded multi-GPU path (csrc/lv_dist.cu) on CPU, without a GPU.

* The library's edge-balanced split (louvain_dist_ranges, a host-only C entry point).
* The host-side transport the library calls back into (paper_conf_ipps_naimmht17_b200.dist.host_comm)
  over gloo, world 2 and 3: rank-major all-gather of bytes, modular uint64 sums.
* The sharding protocol itself, as a model on the plain-C oracle over gloo, world 1-3, BIN_SYNC and
  RELAXED: rank r decides only its range of each bucket against the bucket-start snapshot, the
  moves are all-gathered (padded to the largest owned bucket share, as lv_dist.cu does) and every
  rank commits all of them; Eq. (1)'s L is summed over the ranks' rows.  It must reproduce the
  single-process oracle (b) exactly -- labels, levels, per-level sweeps and exact numerators --
  which is what makes the library's sharded run bit-exact (checked on the GPU in
  tests/test_gpu_parity.py::test_dist_handle_*).
"""
import ctypes
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import graphgen
import oracle
from paper_conf_ipps_naimmht17_b200 import dist_ranges
from paper_conf_ipps_naimmht17_b200.dist import host_comm


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


def _bucket_sizes(engine, p, world):
    """Owned vertices of each bucket on every rank -> the common exchange capacities."""
    sizes = []
    for r, (lo, hi) in enumerate(dist_ranges(engine.rowptr(), world)):
        engine_own = engine.own
        engine.set_owned_range(lo, hi)
        sizes.append([len(engine._bucket(p, b)) for b in range(1, 8)])
        engine.set_owned_range(*engine_own)
    return [max(s[b] for s in sizes) for b in range(7)]


def _exchange(moves, cap, world):
    """Padded all-gather of (v, new) pairs -- the library's k_dist_pack / allgather / k_dist_append."""
    if world == 1:
        return moves
    pad = torch.full((cap, 2), -1, dtype=torch.int32)
    pad[:moves.shape[0]] = moves
    parts = [torch.empty((cap, 2), dtype=torch.int32) for _ in range(world)]
    dist.all_gather(parts, pad)
    allm = torch.cat(parts, dim=0)
    return allm[allm[:, 0] >= 0]


def _sum(x, world):
    if world == 1:
        return x
    t = torch.tensor([x], dtype=torch.int64)
    dist.all_reduce(t)
    return int(t.item())


def model_run_sharded(engine, p, world, rank):
    """The control flow of the library's run_impl on a distributed handle, on the oracle."""
    W = engine.W
    lab = np.arange(engine.n, dtype=np.int32)
    st = {"levels": 0, "sweeps_per_level": [], "num_start": [], "num_end": []}
    cur, Lq, Sq, level = engine, 0, 0, 0
    while True:
        lo, hi = dist_ranges(cur.rowptr(), world)[rank]
        cur.set_owned_range(lo, hi)
        caps = _bucket_sizes(cur, p, world)
        pexp = p.th_bin_exp if cur.n > p.size_limit else p.th_final_exp  # P:330, R14
        if level == 0:
            L_own, Sq, _ = cur.modularity_owned()
            Lq = _sum(L_own, world)
        num_start = Lq * W - Sq
        num_prev, moved_level, sweeps = num_start, 0, 0
        while True:
            cur.begin_sweep()
            moved, pending = 0, []
            for b in range(1, 8):
                if p.mode == 0:
                    allm = _exchange(cur.decide_bucket(p, b), caps[b - 1], world)
                    cur.commit_moves(allm)  # Alg. 1 l.8-11, every rank commits every move
                    moved += int(allm.shape[0])
                else:
                    pending.append(cur.decide_bucket(p, b))
            if p.mode != 0:
                allm = _exchange(torch.cat(pending, dim=0), sum(caps), world)
                cur.commit_moves(allm)
                moved += int(allm.shape[0])
            sweeps += 1
            L_own, S, _ = cur.modularity_owned()
            L = _sum(L_own, world)
            num = L * W - S
            if p.revert_on_decrease and num < num_prev:  # R15
                cur.revert_sweep()
                break
            Lq, Sq = L, S
            moved_level += moved
            if moved == 0 or (num - num_prev) * 10 ** pexp < W * W:  # R13
                break
            num_prev = num
        st["sweeps_per_level"].append(sweeps)
        st["num_start"].append(num_start)
        st["num_end"].append(Lq * W - Sq)
        st["levels"] = level + 1
        if moved_level == 0 or (Lq * W - Sq - num_start) * 10 ** p.th_final_exp < W * W:  # R16
            lab = cur.labels()[lab]
            break
        nxt, mpp = cur.aggregate()
        lab = np.asarray(mpp)[lab]
        cur, level = nxt, level + 1
    st["L"], st["S"] = Lq, Sq
    return lab, st


def _check_against_oracle(name, lab, st, mode=0):
    g = GRAPHS[name]()
    r = oracle.louvain(g, oracle.params(mode=mode))
    assert st["levels"] == r.levels
    assert st["sweeps_per_level"] == r.sweeps_per_level
    assert st["num_start"] == r.num_start and st["num_end"] == r.num_end
    assert np.array_equal(np.asarray(lab), r.labels)
    assert (st["L"], st["S"]) == (r.L, r.S)


def test_dist_ranges_edge_balanced():
    rowptr = np.array([0, 10, 10, 11, 30, 31, 40], dtype=np.int64)
    rs = dist_ranges(rowptr, 3)
    assert rs == [(0, 4), (4, 4), (4, 6)]  # first rows with rowptr >= 13 (row 4) and >= 26 (row 4)
    assert dist_ranges(rowptr, 1) == [(0, 6)]
    # more ranks than vertices: empty ranges are allowed, still a partition
    rs = dist_ranges(np.array([0, 2, 4], dtype=np.int64), 4)
    assert rs[0][0] == 0 and rs[-1][1] == 2 and all(a[1] == b[0] for a, b in zip(rs, rs[1:]))
    rng = np.random.default_rng(0)
    for world in (2, 3, 8):
        deg = rng.integers(0, 50, size=1000)
        rowptr = np.concatenate([[0], np.cumsum(deg)]).astype(np.int64)
        rs = dist_ranges(rowptr, world)
        nnz = int(rowptr[-1])
        for r in range(1, world):  # lower_bound of r*nnz/world, as numpy's searchsorted(side="left")
            assert rs[r][0] == int(np.searchsorted(rowptr, (r * nnz) // world, side="left"))


@pytest.mark.parametrize("name", list(GRAPHS))
def test_world1_model_matches_oracle(name):
    lab, st = model_run_sharded(OracleShard(GRAPHS[name]()), oracle.params(), 1, 0)
    _check_against_oracle(name, lab, st)


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _init(rank, world, port):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)


def _worker(rank, world, port, names, mode, q):
    _init(rank, world, port)
    try:
        out = {}
        for name in names:
            lab, st = model_run_sharded(OracleShard(GRAPHS[name]()), oracle.params(mode=mode), world, rank)
            out[name] = (np.asarray(lab).tolist(), st)
        q.put((rank, out))
    finally:
        dist.destroy_process_group()


def _spawn(target, world, *args):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=target, args=(r, world, port) + args + (q,)) for r in range(world)]
    for pr in procs:
        pr.start()
    results = {}
    for _ in range(world):
        rank, out = q.get(timeout=300)
        results[rank] = out
    for pr in procs:
        pr.join(timeout=60)
        assert pr.exitcode == 0
    return results


@pytest.mark.parametrize("world", [2, 3])
@pytest.mark.parametrize("mode", [0, 1])
def test_gloo_sharded_model_matches_oracle(world, mode):
    names = list(GRAPHS)
    results = _spawn(_worker, world, names, mode)
    for name in names:
        lab0, st0 = results[0][name]
        for r in range(1, world):  # replicas identical on every rank
            assert results[r][name][0] == lab0 and results[r][name][1] == st0
        _check_against_oracle(name, lab0, st0, mode=mode)


def _comm_worker(rank, world, port, q):
    _init(rank, world, port)
    try:
        hc = host_comm()
        # all-gather of bytes, rank-major
        nb = 13
        send = (ctypes.c_uint8 * nb)(*[(rank * 31 + i) % 256 for i in range(nb)])
        recv = (ctypes.c_uint8 * (nb * world))()
        rc1 = hc.allgather(None, ctypes.addressof(send), ctypes.addressof(recv), nb)
        # zero-byte all-gather (an empty bucket on every rank)
        rc0 = hc.allgather(None, ctypes.addressof(send), ctypes.addressof(recv), 0)
        # modular uint64 sum (the delta pass's L change is two's complement)
        vals = (ctypes.c_uint64 * 3)(2 ** 64 - 1 - rank, rank + 1, 2 ** 63 + rank)
        rc2 = hc.allreduce_u64(None, ctypes.addressof(vals), 3)
        q.put((rank, (rc1, rc0, rc2, list(recv), list(vals))))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_host_comm_callbacks_over_gloo(world):
    res = _spawn(_comm_worker, world)
    nb = 13
    want = [(r * 31 + i) % 256 for r in range(world) for i in range(nb)]
    M = 2 ** 64
    sums = [sum((M - 1 - r) for r in range(world)) % M, sum(r + 1 for r in range(world)) % M,
            sum(2 ** 63 + r for r in range(world)) % M]
    for r in range(world):
        rc1, rc0, rc2, recv, vals = res[r]
        assert (rc1, rc0, rc2) == (0, 0, 0)
        assert recv == want
        assert vals == sums
