"""Shared test helpers (golden-file loading, comparison rules of SURVEY.md §8(c) c.2)."""
import json
import os

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
GOLDEN = os.path.join(ROOT, "tests", "golden")


def load_golden(name):
    with open(os.path.join(GOLDEN, name)) as f:
        return json.load(f)


def assert_knn_bitexact(idx, dist, ridx, rdist):
    """Integer-valued inputs: indices and fp32 distances bit-identical."""
    np.testing.assert_array_equal(np.asarray(idx), np.asarray(ridx))
    np.testing.assert_array_equal(np.asarray(dist).view(np.uint32), np.asarray(rdist).view(np.uint32))


def assert_knn_tolerant(Q, T, idx, dist, rdist, rtol=1e-5):
    """Real-valued inputs: per rank |g - o| <= rtol*o
    (exact 0 when o == 0); GPU indices distinct, in range, and the fp64
    recomputed distance of each reported index agrees with the reported one."""
    idx = np.asarray(idx); dist = np.asarray(dist, dtype=np.float64); rdist = np.asarray(rdist, dtype=np.float64)
    nq, k = idx.shape
    assert np.all((idx >= 0) & (idx < T.shape[0]))
    s = np.sort(idx, axis=1)
    assert np.all(s[:, 1:] != s[:, :-1]), "duplicate neighbour index"
    zero = rdist == 0
    assert np.all(dist[zero] == 0), "oracle distance 0 must be reproduced exactly"
    np.testing.assert_array_less(np.abs(dist - rdist), rtol * rdist + 1e-30 + zero * 1.0)
    Qd = np.asarray(Q, dtype=np.float64); Td = np.asarray(T, dtype=np.float64)
    rec = np.sqrt(((Td[idx] - Qd[:, None, :]) ** 2).sum(-1))
    np.testing.assert_array_less(np.abs(rec - dist), rtol * rec + 1e-30 + (rec == 0) * 1e-30 + 1e-37)
