"""Second, independent brute-force KNN for cross-checking the C oracle.

TEST INFRASTRUCTURE ONLY (see oracle/__init__.py). Small inputs only: it
materialises the full [nq, nt] fp64 distance matrix.

Definition (PAPER.md P:L271 output R; Euclidean metric
P:L185): rank every target j of query i by the key (D2(i,j), j) with
D2 = sum_c (Q[i,c] - T[j,c])^2 in fp64, keep the k smallest keys in order.
"""
from __future__ import annotations

import numpy as np


def knn_join_lexsort(Q, T, k):
    Q = np.asarray(Q, dtype=np.float32).astype(np.float64)
    T = np.asarray(T, dtype=np.float32).astype(np.float64)
    nq, nt = Q.shape[0], T.shape[0]
    idx = np.empty((nq, k), dtype=np.int32)
    dist = np.empty((nq, k), dtype=np.float32)
    j = np.arange(nt)
    for i in range(nq):
        diff = T - Q[i][None, :]
        d2 = np.zeros(nt, dtype=np.float64)
        for c in range(Q.shape[1]):  # dimensions in ascending order
            d2 += diff[:, c] * diff[:, c]
        order = np.lexsort((j, d2))[:k]  # primary d2, secondary j
        idx[i] = order
        dist[i] = np.sqrt(d2[order]).astype(np.float32)
    return idx, dist
