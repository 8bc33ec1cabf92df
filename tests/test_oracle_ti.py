"""Pins for oracle/ti.py (the paper's TI-based KNN written out) -- no GPU.

* O3: Eq. 1-4 bound properties on random points (hypothesis) and the equality
  cases on collinear points (closed form).
* P5: the Fig. 5 worked geometry (tests/golden/fig5.json).
* P9: Alg. 2 scan semantics (break / continue / evaluate) on a hand-made list.
* The paper's exactness claim: the TI join equals the brute-force oracle on
  random inputs (integer and real, with ties), and its level-1 results are
  sound (UB >= every member's true k-th distance, every true neighbour's
  cluster is a candidate, P7). Evaluation counts stay within [nq*k, nq*nt].
"""
import math

import numpy as np
import pytest
from hypothesis import given, settings, strategies as st

import oracle
from oracle import ti
from sknn_testutil import load_golden

coord = st.floats(min_value=-1e3, max_value=1e3, allow_nan=False, allow_infinity=False)
pt = st.lists(coord, min_size=3, max_size=3)


@settings(max_examples=300, deadline=None)
@given(pt, pt, pt)
def test_eq1_eq2_bounds(q, t, L):
    d = ti.edist(q, t)
    lb = ti.lb_one_landmark(ti.edist(q, L), ti.edist(t, L))
    ub = ti.ub_one_landmark(ti.edist(q, L), ti.edist(t, L))
    tol = 1e-9 * (1 + ub)
    assert lb <= d + tol
    assert d <= ub + tol


@settings(max_examples=300, deadline=None)
@given(pt, pt, pt, pt)
def test_eq3_eq4_bounds(q, t, L1, L2):
    d = ti.edist(q, t)
    a, D, b = ti.edist(q, L1), ti.edist(L1, L2), ti.edist(L2, t)
    tol = 1e-9 * (1 + a + D + b)
    assert ti.lb_two_landmarks(D, a, b) <= d + tol
    assert d <= ti.ub_two_landmarks(D, a, b) + tol


def test_collinear_equalities():
    # q=0, L=1, t=3 on a line: UB (Eq. 2) = 1 + 2 = 3 = d(q,t); LB with L beyond t
    q, L, t = [0.0], [1.0], [3.0]
    assert ti.ub_one_landmark(ti.edist(q, L), ti.edist(t, L)) == ti.edist(q, t) == 3.0
    L = [5.0]
    assert ti.lb_one_landmark(ti.edist(q, L), ti.edist(t, L)) == 3.0
    # order L1, q, t, L2 on a line: d(L1,L2) = d(L1,q) + d(q,t) + d(t,L2), so LB (Eq. 3) is exact
    L1, q, t, L2 = [0.0], [1.0], [4.0], [6.0]
    assert ti.lb_two_landmarks(ti.edist(L1, L2), ti.edist(q, L1), ti.edist(L2, t)) == 3.0 == ti.edist(q, t)
    # q, L1, L2, t in the order L1 - q ... t - L2 gives the UB (Eq. 4) with equality
    q, L1, L2, t = [1.0], [0.0], [10.0], [8.0]
    # d(q,L1)=1, d(L1,L2)=10, d(L2,t)=2 -> UB = 13 >= d(q,t) = 7; equality needs q-L1-L2-t in order
    assert ti.ub_two_landmarks(ti.edist(L1, L2), ti.edist(q, L1), ti.edist(L2, t)) == 13.0
    q, L1, L2, t = [0.0], [1.0], [4.0], [6.0]
    assert ti.ub_two_landmarks(ti.edist(L1, L2), ti.edist(q, L1), ti.edist(L2, t)) == 6.0 == ti.edist(q, t)


def test_fig5_worked_instance():
    g = load_golden("fig5.json")
    Qm = np.array(g["query_members"], dtype=np.float64)
    Tm = np.array(g["target_members"], dtype=np.float64)
    qc = ti.build_clusters(Qm, np.array([g["cq"]], dtype=np.float64))[0]
    tc = ti.build_clusters(Tm, np.array([g["c1"]], dtype=np.float64))[0]
    assert qc.radius == g["r_q"]
    np.testing.assert_array_equal(tc.dists, g["target_member_dists_desc"])
    assert ti.edist(qc.center, tc.center) == g["D"]
    assert ti.get_ubs(qc, tc, g["k"]) == g["getUBs"]
    assert ti.get_lb(qc, tc) == g["getLB"]
    assert ti.cal_ub(qc, [tc], g["k"]) == g["calUB_single_target_cluster"]
    # the bounds hold for the actual points: every d(q,t) >= getLB, each
    # query's 3rd nearest distance <= calUB
    for q in Qm:
        ds = sorted(ti.edist(q, t) for t in Tm)
        assert ds[0] >= g["getLB"]
        assert ds[2] <= g["calUB_single_target_cluster"]


def test_point_filter_scan_semantics():
    """P9: Alg. 2 lines 9-17 on a hand-made cluster. q2tc = 10, theta = UB = 3:
    members at distances 14 (l=-4 < -3: continue), 12 (l=-2: evaluate),
    9 (l=1: evaluate), 6.5 (l=3.5 > 3: break -> 5 is never looked at)."""
    # 1-D geometry: the center at 0, q at 10; members placed on the line
    T = np.array([[14.0], [12.0], [9.0], [6.5], [5.0]])
    tc = ti.Cluster(center=np.array([0.0]), members=np.arange(5),
                    dists=np.array([14.0, 12.0, 9.0, 6.5, 5.0]), radius=14.0)
    kn, count = ti.point_filter_query(np.array([10.0]), [(0, 0.0)], [tc], T, UB=3.0, k=1)
    assert count == 2  # members 1 and 2 evaluated only
    assert kn[0][1] == 2 and kn[0][0] == 1.0  # nearest is t=9 at distance 1


def _draws(n, m, trials, rng):
    return [rng.choice(n, size=m, replace=False) for _ in range(trials)]


@pytest.mark.parametrize("case", [
    dict(nq=60, nt=90, d=2, k=4, integer=True, self_join=False, seed=0),
    dict(nq=80, nt=80, d=3, k=6, integer=True, self_join=True, seed=1),
    dict(nq=50, nt=120, d=5, k=3, integer=False, self_join=False, seed=2),
    dict(nq=70, nt=70, d=2, k=8, integer=False, self_join=True, seed=3),
    dict(nq=40, nt=40, d=4, k=40, integer=True, self_join=True, seed=4),  # k = nt
])
def test_ti_join_equals_brute_force(case):
    rng = np.random.default_rng(case["seed"])
    mk = (lambda n: rng.integers(0, 7, size=(n, case["d"])).astype(np.float32)) if case["integer"] \
        else (lambda n: rng.standard_normal((n, case["d"])).astype(np.float32))
    T = mk(case["nt"])
    Q = T if case["self_join"] else mk(case["nq"])
    k = case["k"]
    mt = ti.det_lm_num(T.shape[0])
    mq = ti.det_lm_num(Q.shape[0])
    tl, _ = ti.select_landmarks(T, _draws(T.shape[0], mt, 10, rng))
    ql, _ = ti.select_landmarks(Q, _draws(Q.shape[0], mq, 10, rng))
    tcent = T[tl].astype(np.float64)
    qcent = tcent if case["self_join"] else Q[ql].astype(np.float64)
    tcent = ti.lloyd_step(T.astype(np.float64), tcent)  # one Lloyd step (R9)
    if case["self_join"]:
        qcent = tcent
    idx, dist, count, ubs, cands, qcl, tcl = ti.ti_knn_join(Q, T, k, qcent, tcent,
                                                            self_join=case["self_join"])
    bidx, bdist = oracle.knn_join(Q, T, k)
    np.testing.assert_array_equal(idx, bidx)
    np.testing.assert_array_equal(dist, bdist)
    nq, nt = Q.shape[0], T.shape[0]
    assert nq * k <= count <= nq * nt
    # P7 soundness: UB >= every member's true k-th distance; true neighbours'
    # clusters are candidates
    tclus = np.empty(nt, dtype=np.int64)
    for j, c in enumerate(tcl):
        tclus[c.members] = j
    for ci, qc in enumerate(qcl):
        cset = {j for j, _ in cands[ci]}
        for qi in qc.members:
            assert ubs[ci] >= bdist[qi, k - 1] * (1 - 1e-6)
            for t in bidx[qi]:
                assert tclus[t] in cset


def test_landmark_selection_argmax():
    X = np.array([[0.0], [1.0], [2.0], [10.0]])
    draws = [np.array([0, 1]), np.array([0, 3]), np.array([1, 2]), np.array([3, 0])]
    best, sums = ti.select_landmarks(X, draws)
    assert sums == [1.0, 10.0, 1.0, 10.0]
    np.testing.assert_array_equal(best, [0, 3])  # first maximum


def test_det_lm_num():
    assert ti.det_lm_num(434_874) == 1978
    assert ti.det_lm_num(1_000_000) == 3000
    assert ti.det_lm_num(4_000_000) == 6000
    assert ti.det_lm_num(65_554) == 768
    assert ti.det_lm_num(1024) == 96
    assert ti.det_lm_num(60_000) == 734  # the paper prints 745 (reading R10)
    assert ti.det_lm_num(1) == 1


# ------------------------------------------------------------------------
# Hand cases for the clustering helpers and the level-1 pruning direction
# (VERDICT r1 "What's weak" 1): a plausible mistake in each fails one case.

def test_assign_nearest_and_tie_to_lowest_index():
    """assign ("assigns the query point to the closest cluster
    center"): nearest center by Euclidean distance; an exact tie goes to the
    lower center index (R2 applied to centers). Hand-computed on a line."""
    C = np.array([[1.0], [5.0], [8.0]])
    X = np.array([[0.0], [4.0], [9.0], [3.0], [6.5], [100.0]])
    cid, dist = ti.assign(X, C)
    # 3.0 is 2 from c0 and 2 from c1 -> c0; 6.5 is 1.5 from c1 and c2 -> c1
    np.testing.assert_array_equal(cid, [0, 1, 2, 0, 1, 2])
    np.testing.assert_array_equal(dist, [1.0, 1.0, 1.0, 2.0, 1.5, 92.0])
    # the same tie with the center order reversed still picks the lower index
    cid2, _ = ti.assign(np.array([[3.0]]), np.array([[5.0], [1.0]]))
    assert cid2[0] == 0
    # 2-D: (3,4) is 5 from the origin and sqrt(2) from (4,5): not the first center
    cid3, d3 = ti.assign(np.array([[3.0, 4.0]]), np.array([[0.0, 0.0], [4.0, 5.0]]))
    assert cid3[0] == 1 and d3[0] == math.sqrt(2.0)


def test_lloyd_step_mean_and_empty_cluster():
    """lloyd_step (north_star "a few Lloyd iterations", reading R9): the new
    center is the arithmetic mean of the members; an empty cluster keeps its
    center. Hand-computed: {(0,0), (3,0), (0,6)} -> (1, 2)."""
    X = np.array([[0.0, 0.0], [3.0, 0.0], [0.0, 6.0], [20.0, 20.0], [22.0, 24.0]])
    C = np.array([[1.0, 1.0], [100.0, -100.0], [21.0, 21.0]])
    Cn = ti.lloyd_step(X, C)
    np.testing.assert_array_equal(Cn[0], [1.0, 2.0])
    np.testing.assert_array_equal(Cn[1], [100.0, -100.0])   # no member: unchanged
    np.testing.assert_array_equal(Cn[2], [21.0, 22.0])
    # the input centers are not modified in place
    np.testing.assert_array_equal(C[0], [1.0, 1.0])


def test_group_filter_fig5_extension():
    """groupFilter (Alg. 1; Step 2.2 P:L259) on the Fig. 5
    geometry extended by two target clusters. UB = 12.5 (the Fig. 5 calUB).
    c1: LB = 10 - 1 - 2 = 7 <= UB -> kept.
    c2 at (20, 0), radius 0.5: LB = 20 - 1 - 0.5 = 18.5 > UB -> dropped.
    c3 at (0, 14.5), radius 1: LB = 14.5 - 1 - 1 = 12.5 == UB -> kept (R6).
    c4 empty -> skipped. The list holds (j, D) in target-cluster order."""
    g = load_golden("fig5.json")
    Qm = np.array(g["query_members"], dtype=np.float64)
    qc = ti.build_clusters(Qm, np.array([g["cq"]], dtype=np.float64))[0]
    Tm = np.array(g["target_members"] + [[20.0, 0.5], [0.0, 15.5], [0.0, 14.0]], dtype=np.float64)
    cents = np.array([g["c1"], [20.0, 0.0], [0.0, 14.5], [500.0, 500.0]], dtype=np.float64)
    tcl = ti.build_clusters(Tm, cents)
    assert [len(c.members) for c in tcl] == [4, 1, 2, 0]
    assert [c.radius for c in tcl[:3]] == [2.0, 0.5, 1.0]
    UB = g["calUB_single_target_cluster"]
    V = ti.group_filter(UB, qc, tcl)
    assert V == [(0, 10.0), (2, 14.5)]
    # a UB just below the boundary LB drops c3 (the test is LB <= UB, not <)
    V2 = ti.group_filter(12.4, qc, tcl)
    assert V2 == [(0, 10.0)]
    # calUB over all four clusters pools getUBs from every non-empty cluster:
    # getUBs with k: c1 (member distances 0.5, 1, 1.5, 2 closest first) gives
    # 11.5, 12, 12.5, 13 (its first k); c3 (0.5, 1) gives 16, 16.5; c2 gives 21.5
    assert ti.cal_ub(qc, tcl, 3) == 12.5
    assert ti.cal_ub(qc, tcl, 4) == 13.0
    assert ti.cal_ub(qc, tcl, 5) == 16.0
    assert ti.cal_ub(qc, tcl, 7) == 21.5
    assert ti.cal_ub(qc, tcl, 8) == math.inf   # fewer than k bounds pooled
