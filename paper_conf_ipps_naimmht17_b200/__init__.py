"""B200-native GPU Louvain hot path (Naim, Manne, Halappanavar, Tumeo, IPDPS'17).

Thin ctypes binding over ``liblouvain.so`` (C-ABI ``include/louvain.h``):
argument marshalling only -- every step of the method runs in the CUDA kernels
of ``csrc/``.  Accepts numpy arrays (host) or torch CUDA tensors (device);
torch is used only for device memory and streams.  There is no CPU fallback:
importing this package fails loudly if the CUDA library is missing.
"""
from __future__ import annotations

import ctypes
import os
from dataclasses import dataclass
from typing import Optional

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
# LOUVAIN_LIB: an alternative build of the same C-ABI (tools/ab_build.py, A/B measurements)
LIB_PATH = os.environ.get("LOUVAIN_LIB") or os.path.join(_HERE, "liblouvain.so")

OK, E_INVALID_ARG, E_INVALID_GRAPH, E_OVERFLOW, E_NOMEM, E_CUDA, E_NCCL, E_STATE, E_UNSUPPORTED = \
    0, -1, -2, -3, -4, -5, -6, -7, -8
VALIDATE, BORROW, DIST_P2P = 1, 2, 4
MODE_BIN_SYNC, MODE_RELAXED = 0, 1
MAX_LEVELS = 256


class Params(ctypes.Structure):
    _fields_ = [("mode", ctypes.c_int32), ("singleton_rule", ctypes.c_int32),
                ("revert_on_decrease", ctypes.c_int32), ("th_bin_exp", ctypes.c_int32),
                ("th_final_exp", ctypes.c_int32), ("size_limit", ctypes.c_int64),
                ("deg_bounds", ctypes.c_int64 * 6), ("max_sweeps", ctypes.c_int32),
                ("max_levels", ctypes.c_int32)]


class QNum(ctypes.Structure):
    _fields_ = [("L", ctypes.c_uint64), ("S_lo", ctypes.c_uint64), ("S_hi", ctypes.c_uint64),
                ("W", ctypes.c_uint64), ("q", ctypes.c_double)]

    @property
    def S(self) -> int:
        return (int(self.S_hi) << 64) | int(self.S_lo)

    @property
    def num(self) -> int:
        return int(self.L) * int(self.W) - self.S


class Stats(ctypes.Structure):
    _fields_ = [("levels", ctypes.c_int32), ("sweeps", ctypes.c_int32),
                ("n", ctypes.c_int64 * MAX_LEVELS), ("nnz", ctypes.c_int64 * MAX_LEVELS),
                ("sweeps_per_level", ctypes.c_int32 * MAX_LEVELS),
                ("moved_per_level", ctypes.c_int64 * MAX_LEVELS),
                ("num_start", ctypes.c_int64 * MAX_LEVELS), ("num_end", ctypes.c_int64 * MAX_LEVELS),
                ("t_opt_ms", ctypes.c_double * MAX_LEVELS), ("t_agg_ms", ctypes.c_double * MAX_LEVELS),
                ("t_total_ms", ctypes.c_double), ("t_sweep_ms_total", ctypes.c_double),
                ("t_sweep_ms_first", ctypes.c_double), ("t_modularity_ms_total", ctypes.c_double),
                ("edges_swept", ctypes.c_int64), ("moved_first", ctypes.c_int64),
                ("t_sweep_ms_level0", ctypes.c_double * 32),
                ("kernel_launches", ctypes.c_int64), ("cub_calls", ctypes.c_int64), ("q", QNum)]

    def as_dict(self) -> dict:
        lv = self.levels
        return {"levels": lv, "sweeps": self.sweeps, "n": list(self.n[:lv]), "nnz": list(self.nnz[:lv]),
                "sweeps_per_level": list(self.sweeps_per_level[:lv]),
                "moved_per_level": list(self.moved_per_level[:lv]),
                "num_start": list(self.num_start[:lv]), "num_end": list(self.num_end[:lv]),
                "t_opt_ms": list(self.t_opt_ms[:lv]), "t_agg_ms": list(self.t_agg_ms[:lv]),
                "t_total_ms": self.t_total_ms, "t_sweep_ms_total": self.t_sweep_ms_total,
                "t_sweep_ms_first": self.t_sweep_ms_first, "t_modularity_ms_total": self.t_modularity_ms_total,
                "edges_swept": self.edges_swept, "moved_first": self.moved_first,
                "t_sweep_ms_level0": list(self.t_sweep_ms_level0[:min(32, self.sweeps_per_level[0] if lv else 0)]),
                "kernel_launches": self.kernel_launches, "cub_calls": self.cub_calls, "q": self.q.q, "L": int(self.q.L), "S": self.q.S,
                "W": int(self.q.W)}


# host-side transport of the distributed handle (louvain_host_comm_t)
HOST_ALLGATHER = ctypes.CFUNCTYPE(ctypes.c_int32, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_int64)
HOST_ALLREDUCE = ctypes.CFUNCTYPE(ctypes.c_int32, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_int64)


class HostComm(ctypes.Structure):
    _fields_ = [("user", ctypes.c_void_p), ("allgather", HOST_ALLGATHER), ("allreduce_u64", HOST_ALLREDUCE)]


FUNCS = {
    # name: (restype, argtypes)
    "louvain_params_default": (None, [ctypes.POINTER(Params)]),
    "louvain_create_csr": (ctypes.c_int32, [ctypes.c_int64, ctypes.c_int64, ctypes.c_void_p, ctypes.c_void_p,
                                            ctypes.c_void_p, ctypes.c_uint32, ctypes.c_void_p,
                                            ctypes.POINTER(ctypes.c_void_p)]),
    "louvain_destroy": (ctypes.c_int32, [ctypes.c_void_p]),
    "louvain_get_info": (ctypes.c_int32, [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p]),
    "louvain_get_csr": (ctypes.c_int32, [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p]),
    "louvain_set_labels": (ctypes.c_int32, [ctypes.c_void_p, ctypes.c_void_p]),
    "louvain_get_labels": (ctypes.c_int32, [ctypes.c_void_p, ctypes.c_void_p]),
    "louvain_get_totals": (ctypes.c_int32, [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p]),
    "louvain_sweep": (ctypes.c_int32, [ctypes.c_void_p, ctypes.POINTER(Params), ctypes.c_void_p,
                                       ctypes.POINTER(QNum)]),
    "louvain_modularity": (ctypes.c_int32, [ctypes.c_void_p, ctypes.c_void_p, ctypes.POINTER(QNum)]),
    "louvain_aggregate": (ctypes.c_int32, [ctypes.c_void_p, ctypes.POINTER(ctypes.c_void_p), ctypes.c_void_p]),
    "louvain_run": (ctypes.c_int32, [ctypes.c_void_p, ctypes.POINTER(Params), ctypes.c_void_p,
                                     ctypes.POINTER(QNum), ctypes.POINTER(Stats)]),
    "louvain_last_error": (ctypes.c_char_p, []),
    "louvain_launch_counts": (None, [ctypes.c_void_p, ctypes.c_void_p]),
    "louvain_set_owned_range": (ctypes.c_int32, [ctypes.c_void_p, ctypes.c_int64, ctypes.c_int64]),
    "louvain_begin_sweep": (ctypes.c_int32, [ctypes.c_void_p]),
    "louvain_decide_bucket": (ctypes.c_int32, [ctypes.c_void_p, ctypes.POINTER(Params), ctypes.c_int32,
                                               ctypes.c_void_p, ctypes.c_int64, ctypes.POINTER(ctypes.c_int64)]),
    "louvain_commit_moves": (ctypes.c_int32, [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_int64]),
    "louvain_revert_sweep": (ctypes.c_int32, [ctypes.c_void_p]),
    "louvain_compose_labels": (ctypes.c_int32, [ctypes.c_void_p, ctypes.c_int64, ctypes.c_void_p, ctypes.c_void_p]),
    "louvain_modularity_owned": (ctypes.c_int32, [ctypes.c_void_p, ctypes.POINTER(ctypes.c_uint64),
                                                  ctypes.POINTER(ctypes.c_uint64), ctypes.POINTER(ctypes.c_uint64)]),
    "louvain_release_cache": (ctypes.c_int32, []),
    "louvain_dist_unique_id": (ctypes.c_int32, [ctypes.c_void_p]),
    "louvain_create_csr_dist": (ctypes.c_int32, [ctypes.c_int64, ctypes.c_int64, ctypes.c_int64, ctypes.c_void_p,
                                                 ctypes.c_void_p, ctypes.c_void_p, ctypes.c_uint32, ctypes.c_int32,
                                                 ctypes.c_int32, ctypes.c_void_p, ctypes.c_void_p,
                                                 ctypes.POINTER(ctypes.c_void_p)]),
    "louvain_create_csr_dist_host": (ctypes.c_int32, [ctypes.c_int64, ctypes.c_int64, ctypes.c_int64,
                                                      ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p,
                                                      ctypes.c_uint32, ctypes.c_int32, ctypes.c_int32,
                                                      ctypes.POINTER(HostComm), ctypes.c_void_p,
                                                      ctypes.POINTER(ctypes.c_void_p)]),
    "louvain_dist_ranges": (ctypes.c_int32, [ctypes.c_int64, ctypes.c_void_p, ctypes.c_int32, ctypes.c_void_p]),
}

_LIB = None


def lib():
    """The loaded liblouvain.so (raises if it was not built: no fallback)."""
    global _LIB
    if _LIB is None:
        if not os.path.exists(LIB_PATH):
            raise ImportError(f"{LIB_PATH} is missing -- build it with __graft_entry__.build(); "
                              "there is no CPU fallback")
        L = ctypes.CDLL(LIB_PATH)
        for name, (res, args) in FUNCS.items():
            f = getattr(L, name)
            f.restype = res
            f.argtypes = args
        _LIB = L
    return _LIB


class LouvainError(RuntimeError):
    def __init__(self, code: int, msg: str):
        super().__init__(f"louvain error {code}: {msg}")
        self.code = code


def _check(rc: int) -> None:
    if rc != OK:
        raise LouvainError(rc, lib().louvain_last_error().decode(errors="replace"))


def params(**kw) -> Params:
    """Paper defaults with overrides."""
    p = Params()
    lib().louvain_params_default(ctypes.byref(p))
    for k, v in kw.items():
        if k == "deg_bounds":
            for t, b in enumerate(v):
                p.deg_bounds[t] = b
        else:
            setattr(p, k, v)
    return p


def _ptr(x):
    """(address, keepalive) of a numpy array or torch tensor (or None)."""
    if x is None:
        return None, None
    if isinstance(x, np.ndarray):
        x = np.ascontiguousarray(x)
        return x.ctypes.data, x
    if hasattr(x, "data_ptr"):
        if not x.is_contiguous():
            x = x.contiguous()
        return x.data_ptr(), x
    raise TypeError(f"unsupported buffer type {type(x)}")


def _as(x, dtype):
    if x is None:
        return None
    if isinstance(x, np.ndarray):
        return np.ascontiguousarray(x, dtype=dtype)
    import torch
    tmap = {np.int64: torch.int64, np.int32: torch.int32, np.uint32: torch.uint32}
    return x.to(tmap[dtype]).contiguous()


class Graph:
    """One level graph + partition state on the GPU (an opaque C-ABI handle)."""

    def __init__(self, handle: ctypes.c_void_p, stream=None):
        self._h = handle
        self._stream = stream

    @classmethod
    def from_csr(cls, rowptr, col, w=None, validate: bool = False, borrow: bool = False, stream=None) -> "Graph":
        rowptr = _as(rowptr, np.int64)
        col = _as(col, np.int32)
        w = _as(w, np.uint32)
        n = int(rowptr.shape[0]) - 1
        nnz = int(col.shape[0])
        rp, k1 = _ptr(rowptr)
        cp, k2 = _ptr(col)
        wp, k3 = _ptr(w)
        flags = (VALIDATE if validate else 0) | (BORROW if borrow else 0)
        sp = None
        if stream is not None:
            sp = stream.cuda_stream if hasattr(stream, "cuda_stream") else int(stream)
        h = ctypes.c_void_p()
        _check(lib().louvain_create_csr(n, nnz, rp, cp if nnz else None, wp, flags, sp, ctypes.byref(h)))
        g = cls(h, stream)
        g._borrowed = (rowptr, col, w) if borrow else None
        return g

    @classmethod
    def from_csr_dist(cls, n: int, v_begin: int, v_end: int, rowptr_local, col_local, w_local=None, *,
                      rank: int, world: int, comm: str = "nccl", group=None, validate: bool = False,
                      p2p: bool = False, stream=None) -> "Graph":
        """Distributed handle (collective over the `world` ranks of `group`): this rank's rows
        [v_begin, v_end) with global column ids; see include/louvain.h.  comm="nccl": NCCL
        communicator, its unique id broadcast from rank 0 through torch.distributed;
        comm="host": the library's host-side transport over torch.distributed (e.g. gloo).
        p2p=True: commits write every rank's replica through peer memory (CUDA IPC), one
        barrier per bucket instead of the all-gather of moves (LOUVAIN_DIST_P2P)."""
        from . import dist as _dist
        rowptr_local = _as(rowptr_local, np.int64)
        col_local = _as(col_local, np.int32)
        w_local = _as(w_local, np.uint32)
        rp, k1 = _ptr(rowptr_local)
        cp, k2 = _ptr(col_local)
        wp, k3 = _ptr(w_local)
        sp = None
        if stream is not None:
            sp = stream.cuda_stream if hasattr(stream, "cuda_stream") else int(stream)
        flags = (VALIDATE if validate else 0) | (DIST_P2P if p2p else 0)
        h = ctypes.c_void_p()
        keep = None
        if comm == "nccl":
            uid = _dist.nccl_unique_id(rank, group)
            _check(lib().louvain_create_csr_dist(n, v_begin, v_end, rp, cp, wp, flags, rank, world, uid, sp,
                                                 ctypes.byref(h)))
        elif comm == "host":
            keep = _dist.host_comm(group)
            _check(lib().louvain_create_csr_dist_host(n, v_begin, v_end, rp, cp, wp, flags, rank, world,
                                                      ctypes.byref(keep), sp, ctypes.byref(h)))
        else:
            raise ValueError("comm must be 'nccl' or 'host'")
        g = cls(h, stream)
        g._comm_keep = keep  # the callbacks must outlive the handle
        return g

    @classmethod
    def from_host_graph(cls, g, **kw) -> "Graph":
        return cls.from_csr(g.rowptr, g.col, g.w, **kw)

    def close(self) -> None:
        if self._h is not None and self._h.value:
            lib().louvain_destroy(self._h)
        self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()

    # ---------------------------------------------------------------- queries
    def info(self) -> tuple[int, int, int]:
        n, nnz, W = ctypes.c_int64(), ctypes.c_int64(), ctypes.c_uint64()
        _check(lib().louvain_get_info(self._h, ctypes.byref(n), ctypes.byref(nnz), ctypes.byref(W)))
        return n.value, nnz.value, W.value

    @property
    def n(self) -> int:
        return self.info()[0]

    def csr(self):
        n, nnz, _ = self.info()
        rowptr = np.empty(n + 1, dtype=np.int64)
        col = np.empty(max(nnz, 1), dtype=np.int32)
        w = np.empty(max(nnz, 1), dtype=np.uint32)
        _check(lib().louvain_get_csr(self._h, rowptr.ctypes.data, col.ctypes.data, w.ctypes.data))
        return rowptr, col[:nnz], w[:nnz]

    def labels(self, out=None):
        n = self.n
        if out is None:
            out = np.empty(max(n, 1), dtype=np.int32)
        p, keep = _ptr(out)
        _check(lib().louvain_get_labels(self._h, p))
        return out[:n] if isinstance(out, np.ndarray) else out

    def totals(self):
        n = self.n
        a = np.empty(max(n, 1), dtype=np.uint32)
        s = np.empty(max(n, 1), dtype=np.int32)
        _check(lib().louvain_get_totals(self._h, a.ctypes.data, s.ctypes.data))
        return a[:n], s[:n]

    def set_labels(self, labels=None) -> None:
        p, keep = _ptr(_as(labels, np.int32))
        _check(lib().louvain_set_labels(self._h, p))

    # ---------------------------------------------------------------- the method
    def sweep(self, p: Optional[Params] = None, with_q: bool = True):
        """One iteration of Alg. 1's repeat body; returns (moved, QNum or None)."""
        moved = ctypes.c_int64()
        q = QNum()
        _check(lib().louvain_sweep(self._h, ctypes.byref(p or params()), ctypes.byref(moved),
                                   ctypes.byref(q) if with_q else None))
        return moved.value, (q if with_q else None)

    def modularity(self, labels=None) -> QNum:
        p, keep = _ptr(_as(labels, np.int32))
        q = QNum()
        _check(lib().louvain_modularity(self._h, p, ctypes.byref(q)))
        return q

    def aggregate(self, with_map: bool = True, map_out=None):
        """Alg. 3: returns (next Graph, map) -- map in `map_out` (host or device) if given."""
        n = self.n
        if map_out is None and with_map:
            map_out = np.empty(max(n, 1), dtype=np.int32)
        mp, keep = _ptr(map_out)
        h = ctypes.c_void_p()
        _check(lib().louvain_aggregate(self._h, ctypes.byref(h), mp))
        if isinstance(map_out, np.ndarray):
            map_out = map_out[:n]
        return Graph(h, self._stream), map_out

    # ---------------------------------------------------------------- sharded-sweep primitives
    def set_owned_range(self, lo: int, hi: int) -> None:
        _check(lib().louvain_set_owned_range(self._h, lo, hi))

    def begin_sweep(self) -> None:
        _check(lib().louvain_begin_sweep(self._h))

    def decide_bucket(self, p: Params, bucket: int, out) -> int:
        """Moves (v, new) of the owned vertices of `bucket` into out (int32 [cap, 2]); returns count."""
        ptr, keep = _ptr(out)
        cnt = ctypes.c_int64()
        _check(lib().louvain_decide_bucket(self._h, ctypes.byref(p), bucket, ptr, int(out.shape[0]),
                                           ctypes.byref(cnt)))
        return cnt.value

    def commit_moves(self, moves, count: int) -> None:
        ptr, keep = _ptr(moves)
        _check(lib().louvain_commit_moves(self._h, ptr if count else None, count))

    def revert_sweep(self) -> None:
        _check(lib().louvain_revert_sweep(self._h))

    def modularity_owned(self) -> tuple[int, int, int]:
        L, S, W = ctypes.c_uint64(), ctypes.c_uint64(), ctypes.c_uint64()
        _check(lib().louvain_modularity_owned(self._h, ctypes.byref(L), ctypes.byref(S), ctypes.byref(W)))
        return L.value, S.value, W.value


    def run(self, p: Optional[Params] = None, labels_out=None, want_labels: bool = True):
        """Full multilevel Louvain; returns (labels, QNum, stats dict)."""
        n = self.n
        if labels_out is None and want_labels:
            labels_out = np.empty(max(n, 1), dtype=np.int32)
        lp, keep = _ptr(labels_out)
        q = QNum()
        st = Stats()
        _check(lib().louvain_run(self._h, ctypes.byref(p or params()), lp, ctypes.byref(q), ctypes.byref(st)))
        lab = labels_out[:n] if isinstance(labels_out, np.ndarray) else labels_out
        return lab, q, st.as_dict()


def compose_labels(lab, mp, stream=None) -> None:
    """lab[i] = mp[lab[i]] on the device (torch int32 CUDA tensors)."""
    sp = None
    if stream is not None:
        sp = stream.cuda_stream if hasattr(stream, "cuda_stream") else int(stream)
    _check(lib().louvain_compose_labels(lab.data_ptr(), int(lab.numel()), mp.data_ptr(), sp))


def run(rowptr, col, w=None, p: Optional[Params] = None, **kw):
    """One-call convenience: CSR in (host or device), (labels, QNum, stats) out."""
    with Graph.from_csr(rowptr, col, w, **kw) as g:
        return g.run(p)


def release_cache() -> None:
    """Free the device memory kept between handles (scratch cache, idle pool blocks)."""
    _check(lib().louvain_release_cache())


def dist_ranges(rowptr, world: int) -> list[tuple[int, int]]:
    """Edge-balanced contiguous row ranges (host-only C helper, no GPU needed)."""
    rowptr = np.ascontiguousarray(rowptr, dtype=np.int64)
    b = np.zeros(world + 1, dtype=np.int64)
    _check(lib().louvain_dist_ranges(len(rowptr) - 1, rowptr.ctypes.data, world, b.ctypes.data))
    return [(int(b[r]), int(b[r + 1])) for r in range(world)]


def launch_counts() -> tuple[int, int]:
    """Process-wide (kernel launches, CUB calls) of the library so far."""
    k = ctypes.c_int64()
    c = ctypes.c_int64()
    lib().louvain_launch_counts(ctypes.byref(k), ctypes.byref(c))
    return int(k.value), int(c.value)
