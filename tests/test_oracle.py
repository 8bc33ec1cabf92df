"""Pins for the brute-force oracle (oracle/oracle_knn.c) -- no GPU needed.

What pins it:
* P1-P4 hand-computed cases (tests/golden/hand_cases.json), also embedded in
  d=4 with zero padding;
* O1 exhaustive comparison with an independent numpy lexsort brute force and
  with scipy's cKDTree (an independent exact algorithm);
* O2 invariants: sorted rows, self-join rank 0 (reading R3), the prefix
  property, k = nt = full argsort, d = 1 closed form (sorted two-pointer);
* P10 the adversarial equal-norm sphere (ties broken by lowest index).
"""
import numpy as np
import pytest
from scipy.spatial import cKDTree

import oracle
from oracle.ref_numpy import knn_join_lexsort
from sknn_testutil import load_golden
import datagen


@pytest.mark.parametrize("case", load_golden("hand_cases.json")["cases"], ids=lambda c: c["name"])
@pytest.mark.parametrize("pad", [0, 1])
def test_hand_cases(case, pad):
    Q = np.array(case["Q"], dtype=np.float32)
    T = np.array(case["T"], dtype=np.float32)
    if pad:  # embed in d=4 with zero padding: distances unchanged
        Q = np.pad(Q, ((0, 0), (0, 4 - Q.shape[1])))
        T = np.pad(T, ((0, 0), (0, 4 - T.shape[1])))
    idx, dist = oracle.knn_join(Q, T, case["k"])
    np.testing.assert_array_equal(idx, np.array(case["idx"]))
    np.testing.assert_array_equal(dist, np.array(case["dist"], dtype=np.float32))
    if "dist_bits" in case:
        np.testing.assert_array_equal(dist.view(np.uint32), np.array(case["dist_bits"], dtype=np.uint32))


@pytest.mark.parametrize("d", [1, 2, 4, 7, 28])
@pytest.mark.parametrize("seed", [0, 1])
def test_vs_lexsort_and_kdtree(d, seed):
    rng = np.random.default_rng(100 + seed * 10 + d)
    nq, nt = 37, 211
    for integer in (True, False):
        if integer:
            Q = rng.integers(0, 6, size=(nq, d)).astype(np.float32)   # many exact ties
            T = rng.integers(0, 6, size=(nt, d)).astype(np.float32)
        else:
            Q = rng.standard_normal((nq, d)).astype(np.float32)
            T = rng.standard_normal((nt, d)).astype(np.float32)
        for k in (1, 2, 5, 17, nt):
            idx, dist = oracle.knn_join(Q, T, k)
            ridx, rdist = knn_join_lexsort(Q, T, k)
            np.testing.assert_array_equal(idx, ridx)
            np.testing.assert_array_equal(dist, rdist)
        # independent algorithm: KD-tree distances (fp64) agree
        k = 9
        _, dist = oracle.knn_join(Q, T, k)
        kd, _ = cKDTree(T.astype(np.float64)).query(Q.astype(np.float64), k=k)
        np.testing.assert_allclose(dist, kd.reshape(nq, k), rtol=1e-6, atol=1e-6)


def test_all_k_random_small():
    """Exhaustive over k on a tiny input (O1: every k in 1..n)."""
    rng = np.random.default_rng(7)
    X = rng.integers(0, 4, size=(24, 3)).astype(np.float32)
    for k in range(1, 25):
        idx, dist = oracle.knn_join(X, X, k)
        ridx, rdist = knn_join_lexsort(X, X, k)
        np.testing.assert_array_equal(idx, ridx)
        np.testing.assert_array_equal(dist, rdist)


def test_invariants_self_join():
    """O2: sorted rows; self-join rank 0 is distance 0 at the lowest duplicate (R3); prefix property."""
    X = datagen.c3_kegg(600, integer=True)  # 30% duplicate rows
    k = 12
    idx, dist = oracle.knn_join(X, X, k)
    assert np.all(np.diff(dist, axis=1) >= 0)
    assert np.all(dist[:, 0] == 0)
    for i in range(X.shape[0]):
        dup = np.nonzero(np.all(X == X[i], axis=1))[0]
        assert idx[i, 0] == dup.min()
        # all exact duplicates come first, in index order (up to k)
        m = min(k, len(dup))
        np.testing.assert_array_equal(idx[i, :m], dup[:m])
    for kp in (1, 3, 7):
        idx2, dist2 = oracle.knn_join(X, X, kp)
        np.testing.assert_array_equal(idx2, idx[:, :kp])
        np.testing.assert_array_equal(dist2, dist[:, :kp])


def test_full_argsort_k_equals_nt():
    rng = np.random.default_rng(3)
    Q = rng.integers(0, 50, size=(10, 4)).astype(np.float32)
    T = rng.integers(0, 50, size=(64, 4)).astype(np.float32)
    idx, dist = oracle.knn_join(Q, T, 64)
    for i in range(10):
        d2 = ((T.astype(np.int64) - Q[i].astype(np.int64)) ** 2).sum(1)
        order = sorted(range(64), key=lambda j: (d2[j], j))
        np.testing.assert_array_equal(idx[i], order)
        np.testing.assert_array_equal(dist[i], np.sqrt(d2[order]).astype(np.float32))


def test_d1_two_pointer_closed_form():
    """d = 1: the k nearest distances of q are produced by merging outward from
    q's insertion point in the sorted target array (textbook two-pointer)."""
    rng = np.random.default_rng(11)
    T = np.sort(rng.integers(0, 1000, size=300)).astype(np.float32)
    Q = rng.integers(-10, 1010, size=50).astype(np.float32)
    k = 13
    _, dist = oracle.knn_join(Q[:, None], T[:, None], k)
    for i, q in enumerate(Q):
        lo = np.searchsorted(T, q) - 1
        hi = lo + 1
        out = []
        while len(out) < k:
            dl = q - T[lo] if lo >= 0 else np.inf
            dh = T[hi] - q if hi < len(T) else np.inf
            if dl <= dh:
                out.append(dl)
                lo -= 1
            else:
                out.append(dh)
                hi += 1
        np.testing.assert_array_equal(dist[i], np.array(out, dtype=np.float32))


def test_sphere_ties_lowest_index():
    """P10: 384 points at sqrt(30) from the origin plus the origin; a query at
    the origin with k < 385 keeps the origin then the lowest-index sphere points."""
    X = datagen.sphere_ties()
    q = np.zeros((1, 4), np.float32)
    for k in (1, 2, 50, 384, 385):
        idx, dist = oracle.knn_join(q, X, k)
        assert idx[0, 0] == 384 and dist[0, 0] == 0
        np.testing.assert_array_equal(idx[0, 1:], np.arange(k - 1))
        assert np.all(dist[0, 1:] == np.float32(np.sqrt(30.0)))


def test_invalid_args():
    X = np.zeros((4, 2), np.float32)
    with pytest.raises(ValueError):
        oracle.knn_join(X, X, 5)
    with pytest.raises(ValueError):
        oracle.knn_join(X, X, 0)


def test_integer_exactness_bound():
    """Integer workloads keep d * R^2 < 2^24 so squared distances are exact in fp32 (SURVEY c.1)."""
    assert 4 * 255 ** 2 < 2 ** 24
    assert 28 * 700 ** 2 < 2 ** 24
    assert 128 * 255 ** 2 < 2 ** 24
    assert 16 * 1023 ** 2 < 2 ** 24
