"""Independent textbook formulas used to PIN the oracle (never imported by it).

Newman-Girvan modularity written as the dense double sum
    Q = 1/(2m) * sum_{i,j} (A_ij - k_i k_j / (2m)) * delta(c_i, c_j)
with A the stored adjacency (self-loop stored once) and
k_i = sum_j A_ij, evaluated in exact rationals.  This is a different
formula from the oracle's L*W - S numerator form of Eq. (1).
"""
from fractions import Fraction

import numpy as np


def dense_adj(g) -> np.ndarray:
    A = np.zeros((g.n, g.n), dtype=np.int64)
    w = g.weights()
    for i in range(g.n):
        for e in range(g.rowptr[i], g.rowptr[i + 1]):
            A[i, g.col[e]] += int(w[e])
    return A


def q_dense(A: np.ndarray, labels) -> Fraction:
    k = A.sum(axis=1)
    two_m = int(k.sum())
    lab = np.asarray(labels)
    same = lab[:, None] == lab[None, :]
    num = Fraction(int((A * same).sum()), 1) - Fraction(int((np.outer(k, k) * same).sum()), two_m)
    return num / two_m


def q_dense_float_many(A: np.ndarray, label_matrix: np.ndarray) -> np.ndarray:
    """Vectorised float Q for many partitions (rows of label_matrix); brute force only."""
    k = A.sum(axis=1).astype(np.float64)
    two_m = k.sum()
    B = A.astype(np.float64) - np.outer(k, k) / two_m
    out = np.empty(len(label_matrix))
    for t, lab in enumerate(label_matrix):
        same = lab[:, None] == lab[None, :]
        out[t] = (B * same).sum() / two_m
    return out


def set_partitions(n: int):
    """All restricted-growth strings of length n (Bell(n) partitions)."""
    a = [0] * n

    def rec(i, mx):
        if i == n:
            yield list(a)
            return
        for v in range(mx + 2):
            a[i] = v
            yield from rec(i + 1, max(mx, v))

    if n == 0:
        yield []
        return
    yield from rec(1, 0)
