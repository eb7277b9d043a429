"""Vertex-sharded Louvain across ranks (one process per GPU).

Every decision of a degree bucket reads the bucket-start snapshot (Alg. 1
l.6-7), so vertices are independent units inside a bucket:
rank r decides its own vertex range (balanced by edges), the bucket's moves are
all-gathered, and every rank commits all of them to its replica of (C, a_c,
size_c).  The replicas stay bit-identical (integer, order-independent updates);
per sweep the ranks' partial L of Eq. (1) is all-reduced.  Contraction is done
redundantly on every rank (deterministic, identical result), so no graph data
crosses the interconnect.

The control flow is the same as the library's single-GPU driver (`run_impl` in
csrc/lv_engine.cu; exact integer stop tests R13-R16).  The driver is
engine-agnostic: `CudaShard` runs every step in the CUDA kernels through the
C-ABI; the CPU gloo tests plug in an oracle-backed engine to check the
orchestration (partition, exchange, commit, revert) without a GPU.  Collectives
go through torch.distributed (NCCL on GPUs, gloo in tests).
"""
from __future__ import annotations

from typing import Optional

import numpy as np

MAX_MOVES_PER_CALL = None  # capacity is the owned-range size


def edge_balanced_ranges(rowptr: np.ndarray, world: int) -> list[tuple[int, int]]:
    """Contiguous vertex ranges [v_r, v_{r+1}) with rowptr[v_r] ~ r * nnz / world."""
    n = len(rowptr) - 1
    nnz = int(rowptr[-1])
    cuts = [0]
    for r in range(1, world):
        cuts.append(int(np.searchsorted(rowptr, (r * nnz) // world, side="left")))
    cuts.append(n)
    cuts = [min(max(c, 0), n) for c in cuts]
    for r in range(1, len(cuts)):
        cuts[r] = max(cuts[r], cuts[r - 1])
    return [(cuts[r], cuts[r + 1]) for r in range(world)]


class CudaShard:
    """Engine over one C-ABI handle (a level graph on this rank's GPU)."""

    def __init__(self, graph, device=None):
        import torch
        self.g = graph
        self.torch = torch
        self.device = device or torch.device("cuda", torch.cuda.current_device())
        n, nnz, W = graph.info()
        self.n, self.nnz, self.W = n, nnz, W
        self._rowptr = None

    def rowptr(self) -> np.ndarray:
        if self._rowptr is None:
            n = self.n
            rp = np.empty(n + 1, dtype=np.int64)
            import ctypes
            from . import lib, _check
            _check(lib().louvain_get_csr(self.g._h, rp.ctypes.data, None, None))
            self._rowptr = rp
        return self._rowptr

    def set_owned_range(self, lo, hi):
        self.own = (lo, hi)
        self.g.set_owned_range(lo, hi)

    def begin_sweep(self):
        self.g.begin_sweep()

    def decide_bucket(self, p, b):
        lo, hi = self.own
        out = self.torch.empty((max(hi - lo, 1), 2), dtype=self.torch.int32, device=self.device)
        cnt = self.g.decide_bucket(p, b, out)
        return out[:cnt]

    def commit_moves(self, moves):
        if moves.shape[0]:
            self.g.commit_moves(moves.contiguous(), int(moves.shape[0]))

    def revert_sweep(self):
        self.g.revert_sweep()

    def modularity_owned(self):
        return self.g.modularity_owned()

    def aggregate(self):
        mp = self.torch.empty(max(self.n, 1), dtype=self.torch.int32, device=self.device)
        nxt, mp = self.g.aggregate(map_out=mp)
        return CudaShard(nxt, self.device), mp[:self.n]

    def labels(self):
        out = self.torch.empty(max(self.n, 1), dtype=self.torch.int32, device=self.device)
        self.g.labels(out)
        return out[:self.n]

    def new_identity(self, n0):
        return self.torch.arange(n0, dtype=self.torch.int32, device=self.device)

    def compose(self, lab, mp):
        from . import compose_labels
        compose_labels(lab, mp)
        return lab


def _exchange(moves, dist, group, world):
    """All-gather variable-length (v, new) lists; concatenate in rank order."""
    import torch
    if world == 1:
        return moves
    dev = moves.device
    if dist.get_backend(group) == "gloo" and dev.type == "cuda":  # gloo: stage through the host
        return _exchange(moves.cpu(), dist, group, world).to(dev)
    cnt = torch.tensor([moves.shape[0]], dtype=torch.int64, device=dev)
    counts = [torch.zeros(1, dtype=torch.int64, device=dev) for _ in range(world)]
    dist.all_gather(counts, cnt, group=group)
    counts = [int(c.item()) for c in counts]
    m = max(counts)
    if m == 0:
        return moves[:0]
    padded = torch.zeros((m, 2), dtype=moves.dtype, device=dev)
    padded[:moves.shape[0]] = moves
    parts = [torch.empty((m, 2), dtype=moves.dtype, device=dev) for _ in range(world)]
    dist.all_gather(parts, padded, group=group)
    return torch.cat([parts[r][:counts[r]] for r in range(world)], dim=0)


def _allreduce_int(x: int, dist, group, world, device) -> int:
    import torch
    if world == 1:
        return x
    if dist.get_backend(group) == "gloo":
        device = "cpu"
    t = torch.tensor([x], dtype=torch.int64, device=device)
    dist.all_reduce(t, group=group)
    return int(t.item())


def run_sharded(engine, p, group=None, max_levels: int = 256):
    """Multilevel Louvain with the sweep sharded over the ranks of `group`.
    Returns (labels of the input vertices, stats dict) -- identical on every rank."""
    import torch
    import torch.distributed as dist
    if dist.is_available() and dist.is_initialized():
        world = dist.get_world_size(group)
        rank = dist.get_rank(group)
    else:
        world, rank = 1, 0
    W = engine.W
    n0 = engine.n
    lab = engine.new_identity(n0)
    st = {"levels": 0, "sweeps": 0, "n": [], "nnz": [], "sweeps_per_level": [], "moved_per_level": [],
          "num_start": [], "num_end": [], "L": 0, "S": 0, "W": W}
    if W == 0:
        return lab, st
    pw = lambda e: 10 ** e  # noqa: E731
    cur = engine
    Lq = Sq = 0
    level = 0
    dev = getattr(engine, "device", "cpu")
    while True:
        if (p.max_levels > 0 and level >= p.max_levels) or level >= max_levels:
            break
        lo, hi = edge_balanced_ranges(cur.rowptr(), world)[rank]
        cur.set_owned_range(lo, hi)
        pexp = p.th_bin_exp if cur.n > p.size_limit else p.th_final_exp  # P:330, R14
        if level == 0:
            L_own, Sq, _ = cur.modularity_owned()
            Lq = _allreduce_int(L_own, dist, group, world, dev)
        num_start = Lq * W - Sq
        num_prev = num_start
        moved_level = 0
        sweeps = 0
        while True:
            if p.max_sweeps > 0 and sweeps >= p.max_sweeps:
                break
            # level-0 sweep 1 timed on CUDA engines (bench roofline)
            timed = level == 0 and sweeps == 0 and getattr(dev, "type", dev) == "cuda"
            if timed:
                torch.cuda.synchronize()
                ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                ev0.record()
            cur.begin_sweep()
            moved = 0
            pending = []
            for b in range(1, 8):
                allm = _exchange(cur.decide_bucket(p, b), dist, group, world)
                if p.mode == 0:  # BIN_SYNC: commit after each bucket (Alg. 1 l.8-11)
                    cur.commit_moves(allm)
                else:            # RELAXED: one commit per sweep
                    pending.append(allm)
                moved += int(allm.shape[0])
            if p.mode != 0 and pending:
                cur.commit_moves(torch.cat(pending, dim=0))
            if timed:  # device synchronised: every stream's work of the sweep is inside the events
                torch.cuda.synchronize()
                ev1.record()
                ev1.synchronize()
                st["t_sweep_ms_first"] = ev0.elapsed_time(ev1)
                st["moved_first"] = moved
            sweeps += 1
            L_own, S, _ = cur.modularity_owned()
            L = _allreduce_int(L_own, dist, group, world, dev)
            num = L * W - S
            if p.revert_on_decrease and num < num_prev:  # R15
                cur.revert_sweep()
                break
            Lq, Sq = L, S
            moved_level += moved
            if moved == 0 or (num - num_prev) * pw(pexp) < W * W:  # Alg. 1 l.12, R13
                break
            num_prev = num
        num_end = Lq * W - Sq
        st["n"].append(cur.n)
        st["nnz"].append(cur.nnz)
        st["sweeps_per_level"].append(sweeps)
        st["moved_per_level"].append(moved_level)
        st["num_start"].append(num_start)
        st["num_end"].append(num_end)
        st["levels"] = level + 1
        st["sweeps"] += sweeps
        if moved_level == 0 or (num_end - num_start) * pw(p.th_final_exp) < W * W:  # R16
            lab = cur.compose(lab, cur.labels())
            break
        nxt, mp = cur.aggregate()
        lab = cur.compose(lab, mp)
        cur = nxt
        level += 1
    st["L"], st["S"] = Lq, Sq
    st["q"] = (Lq * W - Sq) / float(W) / float(W)
    return lab, st
