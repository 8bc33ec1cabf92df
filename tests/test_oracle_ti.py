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
