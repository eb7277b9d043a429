"""TEST INFRASTRUCTURE ONLY -- ctypes front of the plain C oracle.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s cpu_baseline /
``--impl reference`` leg may import this package.  The product package
(``paper_conf_ipps_naimmht17_b200``) never imports it, and this package
imports nothing from the product.  See ``louvain_oracle.c`` for citations.
"""
from __future__ import annotations

import ctypes
import os
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB = None

BIN_SYNC, RELAXED, SEQ, SEQ_ADAPTIVE = 0, 1, 2, 3
MAX_LEVELS = 256


class Params(ctypes.Structure):
    _fields_ = [("mode", ctypes.c_int32), ("singleton_rule", ctypes.c_int32),
                ("revert_on_decrease", ctypes.c_int32), ("th_bin_exp", ctypes.c_int32),
                ("th_final_exp", ctypes.c_int32), ("size_limit", ctypes.c_int64),
                ("deg_bounds", ctypes.c_int64 * 6), ("max_sweeps", ctypes.c_int32),
                ("max_levels", ctypes.c_int32)]


class Stats(ctypes.Structure):
    _fields_ = [("levels", ctypes.c_int32), ("sweeps", ctypes.c_int32),
                ("n", ctypes.c_int64 * MAX_LEVELS), ("nnz", ctypes.c_int64 * MAX_LEVELS),
                ("sweeps_per_level", ctypes.c_int32 * MAX_LEVELS),
                ("moved_per_level", ctypes.c_int64 * MAX_LEVELS),
                ("num_start", ctypes.c_int64 * MAX_LEVELS), ("num_end", ctypes.c_int64 * MAX_LEVELS),
                ("L", ctypes.c_uint64), ("S", ctypes.c_uint64), ("W", ctypes.c_uint64), ("q", ctypes.c_double)]


def lib():
    global _LIB
    if _LIB is None:
        path = os.path.join(_HERE, "liblouvain_oracle.so")
        if not os.path.exists(path):
            raise RuntimeError(f"{path} missing: run __graft_entry__.build()")
        L = ctypes.CDLL(path)
        vp, i64 = ctypes.c_void_p, ctypes.c_int64
        L.orc_params_default.argtypes = [ctypes.POINTER(Params)]
        L.orc_modularity.argtypes = [i64, vp, vp, vp, vp, vp, vp, vp]
        L.orc_totals.argtypes = [i64, vp, vp, vp, vp, vp]
        L.orc_decide.argtypes = [i64, vp, vp, vp, vp, vp, vp, ctypes.c_uint64, i64, ctypes.c_int32]
        L.orc_decide.restype = ctypes.c_int32
        L.orc_decide_batch.argtypes = [i64, vp, vp, vp, vp, vp, vp, ctypes.c_uint64, ctypes.c_int32, i64, vp, vp]
        L.orc_sweep.argtypes = [i64, vp, vp, vp, ctypes.POINTER(Params), vp, vp, vp, ctypes.c_uint64]
        L.orc_sweep.restype = i64
        L.orc_sweep_counted.argtypes = [i64, vp, vp, vp, ctypes.POINTER(Params), vp, vp, vp, ctypes.c_uint64, vp]
        L.orc_sweep_counted.restype = i64
        L.orc_contract.argtypes = [i64, vp, vp, vp, vp, vp, vp, vp, vp, vp]
        L.orc_contract.restype = i64
        L.orc_louvain.argtypes = [i64, vp, vp, vp, ctypes.POINTER(Params), vp, ctypes.POINTER(Stats)]
        _LIB = L
    return _LIB


def params(**kw) -> Params:
    p = Params()
    lib().orc_params_default(ctypes.byref(p))
    for k, v in kw.items():
        if k == "deg_bounds":
            for t, b in enumerate(v):
                p.deg_bounds[t] = b
        else:
            setattr(p, k, v)
    return p


def _ptr(a):
    return None if a is None else a.ctypes.data


def _g(g):
    rowptr = np.ascontiguousarray(g.rowptr, dtype=np.int64)
    col = np.ascontiguousarray(g.col, dtype=np.int32)
    w = None if g.w is None else np.ascontiguousarray(g.w, dtype=np.uint32)
    return g.n, rowptr, col, w


def modularity(g, C) -> tuple[int, int, int]:
    """Exact (L, S, W) of Eq. (1); Q = (L*W - S) / W^2."""
    n, rowptr, col, w = _g(g)
    C = np.ascontiguousarray(C, dtype=np.int32)
    out = (ctypes.c_uint64 * 3)()
    rc = lib().orc_modularity(n, _ptr(rowptr), _ptr(col), _ptr(w), _ptr(C), ctypes.addressof(out),
                              ctypes.addressof(out) + 8, ctypes.addressof(out) + 16)
    if rc != 0:
        raise OverflowError("W exceeds the int64 guard")
    return int(out[0]), int(out[1]), int(out[2])


def q_of(L: int, S: int, W: int) -> float:
    return (L * W - S) / float(W) / float(W) if W else 0.0


def totals(g, C):
    n, rowptr, col, w = _g(g)
    C = np.ascontiguousarray(C, dtype=np.int32)
    a = np.zeros(max(n, 1), dtype=np.uint64)
    size = np.zeros(max(n, 1), dtype=np.int64)
    lib().orc_totals(n, _ptr(rowptr), _ptr(w), _ptr(C), _ptr(a), _ptr(size))
    return a[:n], size[:n]


def decide(g, C, a, size, W, i, singleton_rule=1) -> int:
    n, rowptr, col, w = _g(g)
    C = np.ascontiguousarray(C, dtype=np.int32)
    a = np.ascontiguousarray(a, dtype=np.uint64)
    size = np.ascontiguousarray(size, dtype=np.int64)
    return int(lib().orc_decide(n, _ptr(rowptr), _ptr(col), _ptr(w), _ptr(C), _ptr(a), _ptr(size), W, i,
                                singleton_rule))


def decide_batch(g, C, a, size, W, verts, singleton_rule=1) -> np.ndarray:
    n, rowptr, col, w = _g(g)
    C = np.ascontiguousarray(C, dtype=np.int32)
    a = np.ascontiguousarray(a, dtype=np.uint64)
    size = np.ascontiguousarray(size, dtype=np.int64)
    verts = np.ascontiguousarray(verts, dtype=np.int64)
    out = np.empty(len(verts), dtype=np.int32)
    lib().orc_decide_batch(n, _ptr(rowptr), _ptr(col), _ptr(w), _ptr(C), _ptr(a), _ptr(size), W,
                           singleton_rule, len(verts), _ptr(verts), _ptr(out))
    return out


class State:
    """Partition state (C, a, size) of one level, updated in place by sweep()."""

    def __init__(self, g, C=None):
        self.g = g
        self.C = np.arange(g.n, dtype=np.int32) if C is None else np.array(C, dtype=np.int32)
        self.a, self.size = totals(g, self.C)
        self.a = np.ascontiguousarray(self.a)
        self.size = np.ascontiguousarray(self.size)
        self.W = int(np.sum(g.weights(), dtype=np.uint64))

    def sweep(self, p: Params) -> int:
        n, rowptr, col, w = _g(self.g)
        return int(lib().orc_sweep(n, _ptr(rowptr), _ptr(col), _ptr(w), ctypes.byref(p), _ptr(self.C),
                                   _ptr(self.a), _ptr(self.size), self.W))

    def sweep_counted(self, p: Params) -> tuple[int, int]:
        """One sweep; returns (moved, D) with D the distinct (vertex, candidate label) pairs evaluated."""
        n, rowptr, col, w = _g(self.g)
        D = ctypes.c_int64()
        moved = int(lib().orc_sweep_counted(n, _ptr(rowptr), _ptr(col), _ptr(w), ctypes.byref(p), _ptr(self.C),
                                            _ptr(self.a), _ptr(self.size), self.W, ctypes.addressof(D)))
        return moved, int(D.value)

    def qnum(self) -> tuple[int, int, int]:
        return modularity(self.g, self.C)


def contract(g, C):
    """Alg. 3: returns (contracted graph, map)."""
    from graphgen import Graph  # input-module dataclass only
    n, rowptr, col, w = _g(g)
    C = np.ascontiguousarray(C, dtype=np.int32)
    nnz = int(rowptr[-1])
    ro = np.zeros(n + 1, dtype=np.int64)
    co = np.zeros(max(nnz, 1), dtype=np.int32)
    wo = np.zeros(max(nnz, 1), dtype=np.uint32)
    mp = np.zeros(max(n, 1), dtype=np.int32)
    nnz2 = ctypes.c_int64()
    n2 = lib().orc_contract(n, _ptr(rowptr), _ptr(col), _ptr(w), _ptr(C), _ptr(ro), _ptr(co), _ptr(wo),
                            ctypes.addressof(nnz2), _ptr(mp))
    m = nnz2.value
    return Graph(int(n2), ro[:n2 + 1].copy(), co[:m].copy(), wo[:m].copy(), None, "contracted"), mp[:n].copy()


@dataclass
class RunResult:
    labels: np.ndarray
    levels: int
    sweeps: int
    n: list
    nnz: list
    sweeps_per_level: list
    moved_per_level: list
    num_start: list
    num_end: list
    L: int
    S: int
    W: int
    q: float


def louvain(g, p: Params | None = None) -> RunResult:
    if p is None:
        p = params()
    n, rowptr, col, w = _g(g)
    labels = np.zeros(max(n, 1), dtype=np.int32)
    st = Stats()
    rc = lib().orc_louvain(n, _ptr(rowptr), _ptr(col), _ptr(w), ctypes.byref(p), _ptr(labels), ctypes.byref(st))
    if rc != 0:
        raise OverflowError("W exceeds the int64 guard")
    lv = st.levels
    return RunResult(labels[:n].copy(), lv, st.sweeps, list(st.n[:lv]), list(st.nnz[:lv]),
                     list(st.sweeps_per_level[:lv]), list(st.moved_per_level[:lv]), list(st.num_start[:lv]),
                     list(st.num_end[:lv]), int(st.L), int(st.S), int(st.W), float(st.q))
