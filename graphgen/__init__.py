"""Seeded synthetic inputs (the one module both the oracle and the CUDA path use).

Holds none of the Louvain method's arithmetic: it only builds CSR graphs
(SURVEY.md 8(d) C1..C5 recipes) through
``libgraphgen.so`` (host builders in C++, device builders in CUDA; the two are
bit-identical) plus small numpy helpers for hand-made weighted test graphs.
"""
from __future__ import annotations

import ctypes
import os
from dataclasses import dataclass, field
from typing import Optional

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB = None


def lib():
    global _LIB
    if _LIB is None:
        path = os.path.join(_HERE, "libgraphgen.so")
        if not os.path.exists(path):
            raise RuntimeError(f"{path} missing: run __graft_entry__.build()")
        L = ctypes.CDLL(path)
        vp, i64, i32, u64, dbl = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int, ctypes.c_uint64, ctypes.c_double
        pp = ctypes.POINTER(ctypes.c_void_p)
        L.gg_karate.argtypes = [pp]
        L.gg_from_edges.argtypes = [i64, i64, vp, vp, i32, pp]
        L.gg_rmat_host.argtypes = [i32, i64, u64, dbl, dbl, dbl, i32, pp]
        L.gg_rmat_device.argtypes = [i32, i64, u64, dbl, dbl, dbl, i32, pp]
        L.gg_mesh3d_host.argtypes = [i32, i32, pp]
        L.gg_mesh3d_device.argtypes = [i32, i32, pp]
        L.gg_rgg_host.argtypes = [i64, dbl, u64, i32, pp]
        L.gg_rgg_device.argtypes = [i64, dbl, u64, i32, pp]
        L.gg_lfr_host.argtypes = [i64, dbl, i32, i32, dbl, i32, i32, dbl, u64, pp]
        for f in ("gg_n", "gg_nnz"):
            getattr(L, f).argtypes = [vp]
            getattr(L, f).restype = i64
        L.gg_on_device.argtypes = [vp]
        L.gg_rowptr.argtypes = [vp]
        L.gg_rowptr.restype = vp
        L.gg_col.argtypes = [vp]
        L.gg_col.restype = vp
        L.gg_labels.argtypes = [vp]
        L.gg_labels.restype = vp
        L.gg_copy_out.argtypes = [vp, vp, vp]
        L.gg_free.argtypes = [vp]
        L.gg_last_error.restype = ctypes.c_char_p
        L.gg_load.argtypes = [ctypes.c_char_p, i32, i32, pp]
        L.gg_save_csrbin.argtypes = [ctypes.c_char_p, i64, i64, vp, vp, vp]
        for f in ("gg_csr_n", "gg_csr_nnz"):
            getattr(L, f).argtypes = [vp]
            getattr(L, f).restype = i64
        for f in ("gg_csr_rowptr", "gg_csr_col", "gg_csr_w"):
            getattr(L, f).argtypes = [vp]
            getattr(L, f).restype = vp
        L.gg_csr_free.argtypes = [vp]
        L.gg_io_last_error.restype = ctypes.c_char_p
        _LIB = L
    return _LIB


@dataclass
class Graph:
    """Host CSR: rowptr int64[n+1], col int32[nnz], w uint32[nnz] or None (unit)."""
    n: int
    rowptr: np.ndarray
    col: np.ndarray
    w: Optional[np.ndarray] = None
    labels: Optional[np.ndarray] = None  # ground truth (LFR) if any
    name: str = ""
    meta: dict = field(default_factory=dict)

    @property
    def nnz(self) -> int:
        return int(self.rowptr[-1]) if self.n >= 0 else 0

    def degrees(self) -> np.ndarray:
        return np.diff(self.rowptr)

    def weights(self) -> np.ndarray:
        return self.w if self.w is not None else np.ones(self.nnz, dtype=np.uint32)


@dataclass
class DeviceGraph:
    """Device CSR as torch tensors (cuda)."""
    n: int
    rowptr: object
    col: object
    name: str = ""
    meta: dict = field(default_factory=dict)

    @property
    def nnz(self) -> int:
        return int(self.col.numel())

    def to_host(self) -> Graph:
        return Graph(self.n, self.rowptr.cpu().numpy(), self.col.cpu().numpy(), None, None, self.name, dict(self.meta))


def _check(rc: int) -> None:
    if rc != 0:
        raise RuntimeError(f"graphgen error {rc}: {lib().gg_last_error().decode()}")


def _take(h: ctypes.c_void_p, name: str, device: bool, meta: dict):
    L = lib()
    try:
        n, nnz = L.gg_n(h), L.gg_nnz(h)
        if device:
            import torch
            rowptr = torch.empty(n + 1, dtype=torch.int64, device="cuda")
            col = torch.empty(max(nnz, 0), dtype=torch.int32, device="cuda")
            _check(L.gg_copy_out(h, rowptr.data_ptr(), col.data_ptr() if nnz else None))
            return DeviceGraph(n, rowptr, col, name, meta)
        rowptr = np.empty(n + 1, dtype=np.int64)
        col = np.empty(nnz, dtype=np.int32)
        _check(L.gg_copy_out(h, rowptr.ctypes.data, col.ctypes.data if nnz else None))
        labels = None
        lp = L.gg_labels(h)
        if lp:
            labels = np.ctypeslib.as_array(ctypes.cast(lp, ctypes.POINTER(ctypes.c_int32)), shape=(n,)).copy()
        return Graph(n, rowptr, col, None, labels, name, meta)
    finally:
        L.gg_free(h)


FORMATS = {"auto": 0, "mtx": 1, "edgelist": 2, "csrbin": 3}


def load(path: str, fmt: str = "auto", one_based: Optional[bool] = None, compact: bool = False) -> Graph:
    """Read a graph file (graph_io.cpp): Matrix Market coordinate (.mtx), edge list
    ("u v [w]" per line) or the binary .csrbin container -> R1 CSR (both directions,
    self-loop once, rows sorted).  w is None for unweighted inputs.  compact=True
    drops isolated vertices with an order-preserving relabel (R21)."""
    L = lib()
    h = ctypes.c_void_p()
    ob = -1 if one_based is None else int(bool(one_based))
    rc = L.gg_load(os.fsencode(path), FORMATS[fmt], ob, ctypes.byref(h))
    if rc != 0:
        raise ValueError(f"graphgen.load({path!r}): {L.gg_io_last_error().decode()}")
    try:
        n, nnz = L.gg_csr_n(h), L.gg_csr_nnz(h)
        rowptr = np.ctypeslib.as_array(ctypes.cast(L.gg_csr_rowptr(h), ctypes.POINTER(ctypes.c_int64)),
                                       shape=(n + 1,)).copy()
        col = np.zeros(0, dtype=np.int32)
        if nnz:
            col = np.ctypeslib.as_array(ctypes.cast(L.gg_csr_col(h), ctypes.POINTER(ctypes.c_int32)),
                                        shape=(nnz,)).copy()
        wp = L.gg_csr_w(h)
        w = None
        if wp and nnz:
            w = np.ctypeslib.as_array(ctypes.cast(wp, ctypes.POINTER(ctypes.c_uint32)), shape=(nnz,)).copy()
    finally:
        L.gg_csr_free(h)
    g = Graph(int(n), rowptr, col, w, None, os.path.basename(path), {"file": path})
    if compact:
        deg = np.diff(g.rowptr)
        keep = np.flatnonzero(deg > 0)
        newid = np.full(g.n, -1, dtype=np.int64)
        newid[keep] = np.arange(len(keep))
        g = Graph(len(keep), np.concatenate([[0], np.cumsum(deg[keep])]).astype(np.int64),
                  newid[g.col].astype(np.int32), g.w, None, g.name, dict(g.meta))
    return g


def save_csrbin(g: Graph, path: str) -> None:
    """Write g as .csrbin (read back bit for bit by load())."""
    rowptr = np.ascontiguousarray(g.rowptr, dtype=np.int64)
    col = np.ascontiguousarray(g.col, dtype=np.int32)
    w = None if g.w is None else np.ascontiguousarray(g.w, dtype=np.uint32)
    rc = lib().gg_save_csrbin(os.fsencode(path), g.n, int(rowptr[-1]), rowptr.ctypes.data,
                              col.ctypes.data if len(col) else None, None if w is None else w.ctypes.data)
    if rc != 0:
        raise OSError(lib().gg_io_last_error().decode())


def karate() -> Graph:
    h = ctypes.c_void_p()
    _check(lib().gg_karate(ctypes.byref(h)))
    return _take(h, "karate", False, {"config": "C1"})


def from_edges(n: int, u, v, compact: bool = True) -> Graph:
    u = np.ascontiguousarray(u, dtype=np.int32)
    v = np.ascontiguousarray(v, dtype=np.int32)
    h = ctypes.c_void_p()
    _check(lib().gg_from_edges(n, len(u), u.ctypes.data, v.ctypes.data, int(compact), ctypes.byref(h)))
    return _take(h, "edges", False, {})


def rmat(scale: int, ntuples: Optional[int] = None, seed: int = 1, a: float = 0.57, b: float = 0.19,
         c: float = 0.19, compact: bool = True, device: bool = False):
    """R-MAT, ``ntuples`` undirected tuples (default 8 * 2^scale, i.e. edge factor 16
    counted as directed entries; SURVEY 8(d) 'edge-factor reading')."""
    if ntuples is None:
        ntuples = 8 << scale
    h = ctypes.c_void_p()
    f = lib().gg_rmat_device if device else lib().gg_rmat_host
    _check(f(scale, ntuples, seed, a, b, c, int(compact), ctypes.byref(h)))
    return _take(h, f"rmat{scale}", device, {"scale": scale, "ntuples": ntuples, "seed": seed})


def mesh3d(L: int, morton: bool = True, device: bool = False):
    h = ctypes.c_void_p()
    f = lib().gg_mesh3d_device if device else lib().gg_mesh3d_host
    _check(f(L, int(morton), ctypes.byref(h)))
    return _take(h, f"mesh{L}", device, {"L": L, "morton": morton})


def rgg(n: int, rfac: float = 0.55, seed: int = 1, compact: bool = True, device: bool = False):
    h = ctypes.c_void_p()
    f = lib().gg_rgg_device if device else lib().gg_rgg_host
    _check(f(n, rfac, seed, int(compact), ctypes.byref(h)))
    return _take(h, f"rgg{n}", device, {"n": n, "rfac": rfac, "seed": seed})


def lfr(n: int = 1_000_000, gamma: float = 2.5, kmin: int = 8, kmax: int = 1000, beta: float = 1.5,
        smin: int = 50, smax: int = 5000, mu: float = 0.3, seed: int = 1) -> Graph:
    h = ctypes.c_void_p()
    _check(lib().gg_lfr_host(n, gamma, kmin, kmax, beta, smin, smax, mu, seed, ctypes.byref(h)))
    return _take(h, f"lfr{n}", False, {"n": n, "mu": mu, "seed": seed})


# ---------------------------------------------------------------- weighted test graphs
def weighted_csr(n: int, u, v, w) -> Graph:
    """Undirected weighted edges (u, v, w>0), no duplicates -> CSR with each non-loop
    edge stored in both directions and each self-loop once."""
    u = np.asarray(u, dtype=np.int64)
    v = np.asarray(v, dtype=np.int64)
    w = np.asarray(w, dtype=np.uint64)
    loop = u == v
    src = np.concatenate([u, v[~loop]])
    dst = np.concatenate([v, u[~loop]])
    ww = np.concatenate([w, w[~loop]])
    order = np.lexsort((dst, src))
    src, dst, ww = src[order], dst[order], ww[order]
    rowptr = np.zeros(n + 1, dtype=np.int64)
    np.add.at(rowptr, src + 1, 1)
    rowptr = np.cumsum(rowptr).astype(np.int64)
    return Graph(n, rowptr, dst.astype(np.int32), ww.astype(np.uint32), None, "weighted")


def random_weighted(n: int, p: float, seed: int, wmax: int = 5, loops: bool = True) -> Graph:
    """Small G(n,p) with integer weights in [1,wmax] and optional self-loops (test inputs)."""
    rng = np.random.default_rng(seed)
    us, vs, ws = [], [], []
    for i in range(n):
        for j in range(i + (0 if loops else 1), n):
            pij = p if i != j else p / 2
            if rng.random() < pij:
                us.append(i); vs.append(j); ws.append(int(rng.integers(1, wmax + 1)))
    return weighted_csr(n, us, vs, ws)


# ---------------------------------------------------------------- named configs
def config(name: str, device: bool = False, seed: int = 1):
    """BASELINE.json configs as concrete inputs; '-small' variants are
    the scaled-down parity cases."""
    if name == "C1":
        return karate()
    if name == "C2":
        return lfr(1_000_000, seed=seed)
    if name == "C2-small":
        return lfr(20_000, seed=seed)
    if name == "C3":
        return rmat(24, seed=seed, device=device)
    if name == "C3-small":
        return rmat(16, seed=seed, device=device)
    if name == "C4a":
        return mesh3d(368, True, device=device)
    if name == "C4a-small":
        return mesh3d(40, True, device=device)
    if name == "C4b":
        return rgg(50_000_000, seed=seed, device=device)
    if name == "C4b-small":
        return rgg(200_000, seed=seed, device=device)
    if name == "C5":
        return rmat(27, seed=seed, device=device)
    raise KeyError(name)
