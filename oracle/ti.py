"""The paper's triangle-inequality (TI) KNN, written out step by step.

TEST INFRASTRUCTURE ONLY (see oracle/__init__.py). Plain fp64 numpy / Python
loops, small inputs only. Every function follows the paper's text in its
order and notation; citations are ``P:L<n>`` = line n of the paper transcript
 with the section / equation / algorithm it falls in.

This module is the second oracle: the TI-based join (Fig. 4 main procedure)
must return exactly the brute-force result of ``oracle.knn_join`` -- that is
the paper's own claim that TI only discards targets that provably cannot be
among the k nearest. tests/test_oracle_ti.py pins it
against brute force, against the paper's worked Fig. 5 geometry, and against
the closed forms of Eq. 1-4.

Readings of the paper used here (DESIGN.md §2 lists them all):
* R2/R4  keys are (squared distance, target index); ties go to the lowest index.
* R6     every prune test keeps the boundary (keep iff bound <= theta).
* R7     fp64 rounding: a relative slack ``ETA64`` is added to every prune test.
* R8     kNearests starts as k placeholders (+inf, -1); theta = min(UB, k-th).
* R11    members of a target cluster are ordered by distance to the center,
         descending, ties by index ascending.
* R12    getUBs uses the k members closest to the center (fewer if the cluster
         is smaller).
"""
from __future__ import annotations

import math
from dataclasses import dataclass, field

import numpy as np

# R7 (fp64 flavour): relative slack for comparisons of sums of computed
# distances. Each fp64 distance has relative error < 1e-15 for d <= 1e3.
ETA64 = 1e-12


def edist(a, b) -> float:
    """Euclidean distance ``Edistance`` (P:L185 metric; Alg. 2 lines 6, 15)."""
    a = np.asarray(a, dtype=np.float64)
    b = np.asarray(b, dtype=np.float64)
    s = 0.0
    for c in range(a.shape[0]):
        diff = float(a[c]) - float(b[c])
        s += diff * diff
    return math.sqrt(s)


def sqdist(a, b) -> float:
    a = np.asarray(a, dtype=np.float64)
    b = np.asarray(b, dtype=np.float64)
    s = 0.0
    for c in range(a.shape[0]):
        diff = float(a[c]) - float(b[c])
        s += diff * diff
    return s


# ---------------------------------------------------------------- Eq. 1-4 --
def lb_one_landmark(d_qL: float, d_tL: float) -> float:
    """Eq. 1 (§II-B): LB(q,t) = |d(q,L) - d(t,L)|."""
    return abs(d_qL - d_tL)


def ub_one_landmark(d_qL: float, d_tL: float) -> float:
    """Eq. 2 (§II-B): UB(q,t) = d(q,L) + d(t,L)."""
    return d_qL + d_tL


def lb_two_landmarks(d_L1L2: float, d_qL1: float, d_L2t: float) -> float:
    """Eq. 3 (Fig. 3): LB(q,t) = d(L1,L2) - d(q,L1) - d(L2,t)."""
    return d_L1L2 - d_qL1 - d_L2t


def ub_two_landmarks(d_L1L2: float, d_qL1: float, d_L2t: float) -> float:
    """Eq. 4 (Fig. 3): UB(q,t) = d(q,L1) + d(L1,L2) + d(L2,t)."""
    return d_qL1 + d_L1L2 + d_L2t


# ------------------------------------------------------- Step 1: clusters --
def det_lm_num(n: int) -> int:
    """detLmNum (§II-C Step 1; §IV-D1): 3*sqrt(n) clusters.

    Reading R10: floor(3*sqrt(n)), at least 1, at most n.
    """
    return max(1, min(n, int(math.floor(3.0 * math.sqrt(n)))))


def landmark_sum(X, idx) -> float:
    """Sum S of all pairwise distances among one candidate landmark set."""
    s = 0.0
    for a in range(len(idx)):
        for b in range(a + 1, len(idx)):
            s += edist(X[idx[a]], X[idx[b]])
    return s


def select_landmarks(X, trial_draws):
    """init: landmark selection (§III-A).

    ``trial_draws`` is the list of candidate index sets the method draws at
    random (one per trial; the paper uses 10 trials of 3*sqrt(n) points). The
    random draws are inputs here. Returns the candidate set with the largest
    pairwise-distance sum S (first trial on ties) and all sums.
    """
    sums = [landmark_sum(X, t) for t in trial_draws]
    best = int(np.argmax(np.asarray(sums)))  # argmax returns the first maximum
    return np.asarray(trial_draws[best]), sums


def assign(X, C):
    """Assign every point to its closest landmark.

    Ties go to the lowest center index. Returns (cluster id, distance).
    """
    n = X.shape[0]
    cid = np.empty(n, dtype=np.int64)
    dist = np.empty(n, dtype=np.float64)
    for i in range(n):
        best, bd = -1, math.inf
        for c in range(C.shape[0]):
            dd = edist(X[i], C[c])
            if dd < bd:
                best, bd = c, dd
        cid[i], dist[i] = best, bd
    return cid, dist


def lloyd_step(X, C):
    """One Lloyd iteration (north_star "a few Lloyd iterations"; reading R9).

    Not in the paper: the paper stops after the landmark sampler. New
    center = mean of the members assigned to it; an empty cluster keeps its
    old center.
    """
    cid, _ = assign(X, C)
    Cn = np.array(C, dtype=np.float64, copy=True)
    for c in range(C.shape[0]):
        m = X[cid == c]
        if m.shape[0] > 0:
            Cn[c] = m.astype(np.float64).mean(axis=0)
    return Cn


@dataclass
class Cluster:
    center: np.ndarray
    members: np.ndarray            # point indices; targets: distance-descending (R11)
    dists: np.ndarray              # distance of each member to the center, same order
    radius: float = 0.0            # maxWithinDist (Alg. 1 line 4)
    extra: dict = field(default_factory=dict)


def build_clusters(X, C):
    """init(Q, T, mq, mt) (§II-C Step 1; §III-A).

    For each cluster: the members, their distances to the center sorted in
    descending order (ties: lower index first, R11) and the maximal member
    distance (radius). The same structure serves query clusters (only the
    radius is used) and target clusters.
    """
    cid, dist = assign(X, C)
    out = []
    for c in range(C.shape[0]):
        mem = np.nonzero(cid == c)[0]
        dd = dist[mem]
        order = np.lexsort((mem, -dd))  # descending distance, then index
        mem, dd = mem[order], dd[order]
        out.append(Cluster(center=np.asarray(C[c], dtype=np.float64), members=mem,
                           dists=dd, radius=float(dd[0]) if len(dd) else 0.0))
    return out


# ------------------------------------------- Step 2: level-1 (cluster) filter --
def get_ubs(qc: Cluster, tc: Cluster, k: int):
    """getUBs(q, t, k) (Fig. 5; Fig. 4).

    With a the query member farthest from c_q (distance r_q) and u, v, w, ...
    the k target members closest to c_t: the i-th bound is
    d(a,c_q) + d(c_q,c_t) + d(c_t,u_i)  (Eq. 4, 2-landmark UB).
    A cluster with fewer than k members contributes all of them (R12).
    """
    D = edist(qc.center, tc.center)
    closest = np.sort(tc.dists)[:k]  # members closest to the landmark
    return [ub_two_landmarks(D, qc.radius, float(x)) for x in closest]


def cal_ub(qc: Cluster, tclusters, k: int) -> float:
    """calUB(q, C, k) (§II-C Step 2.1; Fig. 4).

    Pool the getUBs bounds of every target cluster, return the k-th smallest.
    (The footnote's early termination, does not change the value.)
    """
    W = []
    for tc in tclusters:
        if len(tc.members):
            W.extend(get_ubs(qc, tc, k))
    W.sort()
    return W[k - 1] if len(W) >= k else math.inf


def get_lb(qc: Cluster, tc: Cluster) -> float:
    """getLB(q, t) (P:L259 Step 2.2; Fig. 4): d(c_q,c_t) - r_q - r_t."""
    return lb_two_landmarks(edist(qc.center, tc.center), qc.radius, tc.radius)


def group_filter(UB: float, qc: Cluster, tclusters):
    """groupFilter(UB, q, C) (Fig. 4; Alg. 1).

    Keep target cluster j iff its lower bound l satisfies l <= UB (reading
    R6: the text prunes only if UB < l). Empty clusters are skipped.
    Returns the candidate list [(j, d(c_q, c_j))] in target-cluster order.
    """
    V = []
    for j, tc in enumerate(tclusters):
        if not len(tc.members):
            continue
        l = get_lb(qc, tc)
        if l <= UB + ETA64 * (abs(l) + UB):
            V.append((j, edist(qc.center, tc.center)))
    return V


# ------------------------------------------- Step 3: level-2 (point) filter --
def point_filter_query(q_point, cands, tclusters, T, UB: float, k: int):
    """pointFilter for one query point (Fig. 4; Alg. 2).

    cands: [(j, D_j)] already sorted by D_j ascending (Fig. 4 line 1).
    Returns (sorted [(d2, t)] of length k, number of distance evaluations).
    """
    kn = [(math.inf, -1)] * k            # kNearests (R8 placeholders)
    theta = UB                            # Alg. 2 line 3
    count = 0
    for j, _D in cands:                   # Alg. 2 line 5
        tc = tclusters[j]
        q2tc = edist(q_point, tc.center)  # Alg. 2 line 6
        for pos in range(len(tc.members)):  # line 7, members distance-descending
            t = int(tc.members[pos])
            q2t_lb = q2tc - float(tc.dists[pos])          # line 9 (Eq. 1 signed)
            slack = ETA64 * (abs(q2tc) + float(tc.dists[pos]) + theta)
            if q2t_lb > theta + slack:                     # line 10
                break                                      # line 11
            elif q2t_lb < -theta - slack:                  # line 12
                continue                                   # line 13
            d2 = sqdist(q_point, T[t])                     # line 15
            count += 1
            key = (d2, t)
            if key < kn[-1]:                               # line 16
                kn[-1] = key
                kn.sort()
                theta = min(UB, math.sqrt(kn[-1][0]))      # line 17 (R8)
    return kn, count


def ti_knn_join(Q, T, k: int, q_centers, t_centers, self_join: bool = False):
    """Main procedure of TI-based KNN (Fig. 4), given the landmarks.

    Steps: init (build clusters on Q and T), then for each query cluster:
    calUB -> groupFilter -> pointFilter. Returns (idx [nq,k], dist [nq,k],
    evaluation count, per-query-cluster UB list, candidate lists).
    """
    Q = np.asarray(Q, dtype=np.float32).astype(np.float64)
    T = np.asarray(T, dtype=np.float32).astype(np.float64)
    tcl = build_clusters(T, np.asarray(t_centers, dtype=np.float64))
    qcl = tcl if self_join else build_clusters(Q, np.asarray(q_centers, dtype=np.float64))
    nq = Q.shape[0]
    idx = np.full((nq, k), -1, dtype=np.int32)
    dist = np.full((nq, k), np.inf, dtype=np.float32)
    total = 0
    ubs, cand_lists = [], []
    for qc in qcl:
        if not len(qc.members):
            ubs.append(math.inf)
            cand_lists.append([])
            continue
        UB = cal_ub(qc, tcl, k)
        cands = group_filter(UB, qc, tcl)
        cands.sort(key=lambda x: (x[1], x[0]))  # ascending center distance
        ubs.append(UB)
        cand_lists.append(cands)
        for qi in qc.members:
            kn, cnt = point_filter_query(Q[qi], cands, tcl, T, UB, k)
            total += cnt
            for r, (d2, t) in enumerate(kn):
                idx[qi, r] = t
                dist[qi, r] = np.float32(math.sqrt(d2))
    return idx, dist, total, ubs, cand_lists, qcl, tcl
