"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle.

Bar (SURVEY.md §8(c) c.2 / north_star): integer-valued inputs bit-exact
(indices and fp32 distances); real-valued inputs within 1e-5 relative with
neighbour sets equal up to ties (sknn_testutil.assert_knn_tolerant).
Inputs come from datagen (seeded); expected values only from oracle/.
"""
import os

import numpy as np
import pytest

import datagen
import oracle
from sknn_testutil import assert_knn_bitexact, assert_knn_tolerant

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")


@pytest.fixture(scope="module")
def sknn():
    import paper_conf_icde_chends17_b200 as s
    from paper_conf_icde_chends17_b200 import buildlib
    buildlib.build()
    assert torch.cuda.is_available(), "GPU tests need a CUDA device"
    return s


def dev(x):
    return torch.from_numpy(np.ascontiguousarray(x, dtype=np.float32)).cuda()


def run(sknn, Q, T, k, self_join, **opts):
    dQ = dev(Q)
    dT = dQ if self_join else dev(T)
    idx, dist, st = sknn.join(dQ, dT, k, stats=True, **opts)
    torch.cuda.synchronize()
    return idx.cpu().numpy(), dist.cpu().numpy(), st


CASES_INT = [
    ("C1", 1.0), ("C3int", 0.05), ("C4", 0.004), ("C5", 0.0025),
]


@pytest.mark.parametrize("path,mapping", [("auto", "auto"), ("sparse", "thread"), ("sparse", "warp"),
                                          ("brute", "auto")])
def test_c1_bitexact_all_paths(sknn, path, mapping):
    Q, T, k, sj = datagen.workload("C1")
    idx, dist, st = run(sknn, Q, T, k, sj, force_path=path, mapping=mapping)
    ridx, rdist = oracle.knn_join(Q, T, k)
    assert_knn_bitexact(idx, dist, ridx, rdist)
    if path != "brute":
        assert 0 < st["pruned_pct"] < 100


@pytest.mark.parametrize("name,scale", CASES_INT)
@pytest.mark.parametrize("mapping", ["auto", "thread", "warp"])
def test_integer_workloads_bitexact(sknn, name, scale, mapping):
    Q, T, k, sj = datagen.workload(name, scale)
    idx, dist, st = run(sknn, Q, T, k, sj, mapping=mapping)
    ridx, rdist = oracle.knn_join(Q, T, k)
    assert_knn_bitexact(idx, dist, ridx, rdist)
    assert st["dist_evals"] >= Q.shape[0] * k


@pytest.mark.parametrize("name,scale", [("C2", 0.05), ("C3", 0.1)])
@pytest.mark.parametrize("mapping", ["thread", "warp"])
def test_real_workloads_tolerant(sknn, name, scale, mapping):
    Q, T, k, sj = datagen.workload(name, scale)
    idx, dist, st = run(sknn, Q, T, k, sj, mapping=mapping)
    _, rdist = oracle.knn_join(Q, T, k)
    assert_knn_tolerant(Q, T, idx, dist, rdist)


def test_sphere_ties(sknn):
    """P10: equal-norm sphere + origin, queries at the origin and at sphere points."""
    X = datagen.sphere_ties()
    Q = np.concatenate([np.zeros((3, 4), np.float32), X[:40]], axis=0)
    for k in (1, 5, 17, 32):
        for path in ("auto", "brute"):
            for mapping in ("thread", "warp"):
                idx, dist, _ = run(sknn, Q, X, k, False, force_path=path, mapping=mapping)
                ridx, rdist = oracle.knn_join(Q, X, k)
                assert_knn_bitexact(idx, dist, ridx, rdist)


@pytest.mark.parametrize("d", [1, 2, 3, 5, 7, 13, 33, 64])
def test_odd_dimensions(sknn, d):
    rng = np.random.default_rng(d)
    T = rng.integers(0, 40, size=(3000, d)).astype(np.float32)
    Q = rng.integers(0, 40, size=(700, d)).astype(np.float32)
    for k in (1, 9, 32):
        for mapping in ("thread", "warp"):
            idx, dist, _ = run(sknn, Q, T, k, False, mapping=mapping)
            ridx, rdist = oracle.knn_join(Q, T, k)
            assert_knn_bitexact(idx, dist, ridx, rdist)


@pytest.mark.parametrize("n,k", [(1, 1), (2, 2), (5, 5), (33, 32), (100, 32), (257, 3)])
def test_tiny_and_k_equals_n(sknn, n, k):
    rng = np.random.default_rng(n)
    X = rng.integers(0, 5, size=(n, 3)).astype(np.float32)
    for mapping in ("thread", "warp"):
        idx, dist, _ = run(sknn, X, X, k, True, mapping=mapping)
        ridx, rdist = oracle.knn_join(X, X, k)
        assert_knn_bitexact(idx, dist, ridx, rdist)


def test_all_duplicates(sknn):
    """Degenerate: every point identical -> one cluster, all distances 0, lowest indices."""
    X = np.full((2000, 4), 7.0, np.float32)
    idx, dist, _ = run(sknn, X, X, 16, True)
    assert np.all(dist == 0)
    assert np.all(idx == np.arange(16)[None, :])


def test_big_cluster_sort_path(sknn):
    """A cluster larger than the 4096-key shared-memory sort (k_segsort_big)."""
    rng = np.random.default_rng(5)
    big = rng.integers(0, 3, size=(20000, 2)).astype(np.float32)   # dense blob
    far = rng.integers(1000, 1100, size=(500, 2)).astype(np.float32)
    X = np.concatenate([big, far])
    idx, dist, _ = run(sknn, X, X, 8, True, n_clusters_t=4)
    ridx, rdist = oracle.knn_join(X, X, 8)
    assert_knn_bitexact(idx, dist, ridx, rdist)


def test_host_pointers_match_device(sknn):
    Q, T, k, sj = datagen.workload("C1")
    hidx, hdist = sknn.join(Q, Q, k)     # numpy host buffers: staged inside the call
    didx, ddist, _ = run(sknn, Q, T, k, sj)
    np.testing.assert_array_equal(hidx, didx)
    np.testing.assert_array_equal(hdist, ddist)


def test_without_indices(sknn):
    Q, T, k, sj = datagen.workload("C1")
    dQ = dev(Q)
    idx, dist = sknn.join(dQ, dQ, k, with_index=False)
    assert idx is None
    _, rdist = oracle.knn_join(Q, T, k)
    np.testing.assert_array_equal(dist.cpu().numpy(), rdist)


def test_seed_and_lloyd_do_not_change_results(sknn):
    Q, T, k, sj = datagen.workload("C3int", 0.03)
    ridx, rdist = oracle.knn_join(Q, T, k)
    for seed, lloyd, ncl in [(1, 0, 0), (2, 1, 0), (3, 4, 0), (4, 2, 7), (5, 2, 1)]:
        idx, dist, _ = run(sknn, Q, T, k, sj, seed=seed, lloyd_iters=lloyd, n_clusters_t=ncl)
        assert_knn_bitexact(idx, dist, ridx, rdist)


def test_index_build_query_and_invariants(sknn):
    """sknn_build / sknn_query, plus index invariants P6."""
    T = datagen.c5_blobs(30000, which="T")
    Q = datagen.c5_blobs(5000, which="Q")
    k = 32
    ix = sknn.build(dev(T))
    e = ix.export()
    off, orig, dist, cent, rad = e["off"], e["orig"], e["dist"], e["centers"], e["radius"]
    m = len(rad)
    assert off[0] == 0 and off[-1] == T.shape[0] and np.all(np.diff(off) >= 0)
    assert np.array_equal(np.sort(orig), np.arange(T.shape[0]))   # every point exactly once
    for c in range(m):
        seg = dist[off[c]:off[c + 1]]
        if len(seg) == 0:
            assert rad[c] == 0
            continue
        assert np.all(np.diff(seg) <= 0)                         # descending (R11)
        assert rad[c] == seg[0]
        mem = orig[off[c]:off[c + 1]]
        rec = np.sqrt(((T[mem].astype(np.float64) - cent[c, :16].astype(np.float64)) ** 2).sum(1))
        np.testing.assert_allclose(seg, rec, rtol=2e-6)           # recorded distances are exact-ish
        eq = seg[1:] == seg[:-1]
        assert np.all(mem[1:][eq] > mem[:-1][eq])                 # ties by index ascending
    idx, dd, st = ix.query(dev(Q), k, stats=True)
    torch.cuda.synchronize()
    ridx, rdist = oracle.knn_join(Q, T, k)
    assert_knn_bitexact(idx.cpu().numpy(), dd.cpu().numpy(), ridx, rdist)
    ix.close()


def test_level1_soundness(sknn):
    """P7: UB_qc >= the true k-th distance of every member query; the cluster of
    every true neighbour is a candidate of the query's cluster."""
    T = datagen.c5_blobs(20000, which="T")
    Q = datagen.c5_blobs(3000, which="Q")
    k = 32
    ix = sknn.build(dev(T))
    e = ix.export()
    tcl = np.empty(T.shape[0], np.int64)
    for c in range(len(e["radius"])):
        tcl[e["orig"][e["off"][c]:e["off"][c + 1]]] = c
    l1 = ix.debug_level1(dev(Q), k)
    ridx, rdist = oracle.knn_join(Q, T, k)
    qc = l1["q_cluster"]
    assert np.all(l1["ub"][qc] >= rdist[:, -1])
    for i in range(Q.shape[0]):
        cands = set(l1["cand"][qc[i], :l1["cand_count"][qc[i]]].tolist())
        assert set(tcl[ridx[i]].tolist()) <= cands
    ix.close()


def test_merge_partials_equals_unsharded(sknn):
    """Simulated target sharding on one GPU (P11): per-shard partial lists with
    global indices merged by sknn_merge_partials == the unsharded join."""
    T = datagen.c5_blobs(24000, which="T")
    Q = datagen.c5_blobs(4000, which="Q")
    k = 32
    dQ = dev(Q)
    parts_i, parts_d = [], []
    P = 3
    bounds = np.linspace(0, T.shape[0], P + 1).astype(int)
    for r in range(P):
        Ts = dev(T[bounds[r]:bounds[r + 1]])
        i, d = sknn.join(dQ, Ts, k, out_squared=1, index_base=int(bounds[r]))
        parts_i.append(i)
        parts_d.append(d)
    idx, dist = sknn.merge_partials(torch.stack(parts_i), torch.stack(parts_d), k)
    torch.cuda.synchronize()
    ridx, rdist = oracle.knn_join(Q, T, k)
    assert_knn_bitexact(idx.cpu().numpy(), dist.cpu().numpy(), ridx, rdist)


@pytest.mark.slow
def test_c2_full_size_sampled(sknn):
    """C2 at BASELINE size in the launch configuration bench.py times; the oracle
    checks a seeded sample of queries one by one."""
    Q, T, k, sj = datagen.workload("C2")
    idx, dist, st = run(sknn, Q, T, k, sj)
    rng = np.random.default_rng(99)
    s = rng.choice(Q.shape[0], 2000, replace=False)
    _, rdist = oracle.knn_join(Q[s], T, k)
    assert_knn_tolerant(Q[s], T, idx[s], dist[s], rdist)
    assert st["pruned_pct"] > 99.0


@pytest.mark.slow
@pytest.mark.parametrize("name,nsample", [("C3", 3000), ("C3int", 3000), ("C4", 400), ("C5", 400)])
def test_full_size_sampled(sknn, name, nsample):
    """C3 / C4 / C5 at BASELINE.json's full sizes in the launch configuration
    `bench.py --config` times (auto path: elastic switch, dense tiles, split
    tasks); the oracle checks a seeded sample of query rows one by one.
    Integer-valued workloads bit-exact, real-valued within 1e-5 (c.2)."""
    Q, T, k, sj = datagen.workload(name)
    idx, dist, st = run(sknn, Q, T, k, sj)
    rng = np.random.default_rng(7)
    s = np.sort(rng.choice(Q.shape[0], nsample, replace=False))
    ridx, rdist = oracle.knn_join(Q[s], T, k)
    if name == "C3":
        assert_knn_tolerant(Q[s], T, idx[s], dist[s], rdist)
    else:
        assert_knn_bitexact(idx[s], dist[s], ridx, rdist)
    # every row is a sorted, duplicate-free list of in-range indices
    assert np.all(np.diff(dist, axis=1) >= 0)
    assert np.all((idx >= 0) & (idx < T.shape[0]))
    nq, nt = Q.shape[0], T.shape[0]
    assert nq * k <= st["dist_evals"] <= nq * nt


# ------------------------------------------------------------ dense tiles --
@pytest.mark.parametrize("name,scale", [("C1", 1.0), ("C3int", 0.05), ("C4", 0.004), ("C5", 0.0025)])
@pytest.mark.parametrize("mapping", ["thread", "warp"])
def test_dense_tiles_bitexact(sknn, name, scale, mapping):
    """S11: every surviving cluster pair through the tcgen05 dense-tile screen
    (force_path=dense) -- results must stay bit-identical to the oracle."""
    Q, T, k, sj = datagen.workload(name, scale)
    idx, dist, st = run(sknn, Q, T, k, sj, force_path="dense", mapping=mapping)
    ridx, rdist = oracle.knn_join(Q, T, k)
    assert_knn_bitexact(idx, dist, ridx, rdist)
    assert st["dense_pairs"] > 0 and st["dist_evals_dense"] > 0
    assert st["dist_evals_sparse"] == 0


@pytest.mark.parametrize("name,scale", [("C2", 0.05), ("C3", 0.1)])
def test_dense_tiles_real_tolerant(sknn, name, scale):
    Q, T, k, sj = datagen.workload(name, scale)
    idx, dist, st = run(sknn, Q, T, k, sj, force_path="dense")
    _, rdist = oracle.knn_join(Q, T, k)
    assert_knn_tolerant(Q, T, idx, dist, rdist)
    assert st["dense_pairs"] > 0


def test_dense_tiles_ties_and_dims(sknn):
    X = datagen.sphere_ties()
    Q = np.concatenate([np.zeros((3, 4), np.float32), X[:40]], axis=0)
    for k in (1, 17, 32):
        idx, dist, _ = run(sknn, Q, X, k, False, force_path="dense")
        ridx, rdist = oracle.knn_join(Q, X, k)
        assert_knn_bitexact(idx, dist, ridx, rdist)
    rng = np.random.default_rng(17)
    for d in (3, 16, 33, 100, 130):
        T = rng.integers(0, 40, size=(2500, d)).astype(np.float32)
        Qd = rng.integers(0, 40, size=(300, d)).astype(np.float32)
        idx, dist, _ = run(sknn, Qd, T, 9, False, force_path="dense")
        ridx, rdist = oracle.knn_join(Qd, T, 9)
        assert_knn_bitexact(idx, dist, ridx, rdist)


def test_auto_switch_mixes_paths(sknn):
    """The elastic switch (auto) on a dp >= 16 workload sends some pairs to
    dense tiles and the rest to the sparse scan; results stay exact."""
    Q, T, k, sj = datagen.workload("C4", 0.01)
    idx, dist, st = run(sknn, Q, T, k, sj)
    ridx, rdist = oracle.knn_join(Q, T, k)
    assert_knn_bitexact(idx, dist, ridx, rdist)
    assert st["dense_pairs"] > 0 and st["dist_evals_sparse"] > 0
    assert st["dense_pairs"] < st["cand_pairs"]


# ------------------------------------------------------------ multi-GPU --
@pytest.mark.parametrize("policy", [0, 1])
@pytest.mark.parametrize("name,scale,P", [("C3int", 0.05, 3), ("C4", 0.004, 4), ("C5", 0.0025, 8), ("C1", 1.0, 5)])
def test_query_shard_option_covers_all_rows(sknn, policy, name, scale, P):
    """Query sharding (sknn_options.shard_rank/count): P ranks' shards, run one
    after the other into the same output, reproduce the single join
    bit-exactly (P11), for the interleaved (c % P) and the balanced (snake deal
    by the level-1 work estimate) ownership; every row is written by exactly
    one rank (a row another rank owns stays at its -1 fill), and with the
    balanced policy the C4 shards include elastic-switch dense tiles."""
    Q, T, k, sj = datagen.workload(name, scale)
    dQ = dev(Q)
    dT = dQ if sj else dev(T)
    idx = torch.full((Q.shape[0], k), -1, dtype=torch.int32, device="cuda")
    dst = torch.zeros((Q.shape[0], k), dtype=torch.float32, device="cuda")
    owner = np.full(Q.shape[0], -1)
    for r in range(P):
        i1 = torch.full((Q.shape[0], k), -1, dtype=torch.int32, device="cuda")
        d1 = torch.zeros((Q.shape[0], k), dtype=torch.float32, device="cuda")
        sknn.join(dQ, dT, k, out=(i1, d1), shard_rank=r, shard_count=P, shard_policy=policy)
        rows = (i1[:, 0] >= 0).cpu().numpy()
        assert (owner[rows] == -1).all()   # no row computed by two ranks
        owner[rows] = r
        idx[rows] = i1[rows]
        dst[rows] = d1[rows]
    torch.cuda.synchronize()
    assert (owner >= 0).all()
    ridx, rdist = oracle.knn_join(Q, T, k)
    assert_knn_bitexact(idx.cpu().numpy(), dst.cpu().numpy(), ridx, rdist)


def test_dist_nccl_world1(sknn):
    """The torch.distributed orchestration on the NCCL backend (world size 1 on
    the one GPU the driver provides): both sharding modes equal the join."""
    import os
    import socket
    import torch.distributed as tdist
    from paper_conf_icde_chends17_b200 import dist as sdist
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    tdist.init_process_group("nccl", rank=0, world_size=1, device_id=torch.device("cuda", 0))
    try:
        T = datagen.c5_blobs(20000, which="T")
        Q = datagen.c5_blobs(3000, which="Q")
        k = 32
        ridx, rdist = oracle.knn_join(Q, T, k)
        i, d = sdist.join_target_sharded(dev(Q), dev(T), k, 0)
        assert_knn_bitexact(i.cpu().numpy(), d.cpu().numpy(), ridx, rdist)
        i, d = sdist.join_target_sharded(dev(Q), dev(T), k, 0, exchange="all_to_all")
        assert_knn_bitexact(i.cpu().numpy(), d.cpu().numpy(), ridx, rdist)
        i, d = sdist.join_query_sharded(dev(Q), dev(T), k, self_join=False)
        assert_knn_bitexact(i.cpu().numpy(), d.cpu().numpy(), ridx, rdist)
        # the fused peer-memory merge's path on a world of one: symmetric-memory
        # buffers, device barrier, merge kernel reading the (here local) buffer
        try:
            import torch.distributed._symmetric_memory as symm_mem
            symm_mem.empty((4,), dtype=torch.float32, device="cuda")
            peer_ok = True
        except Exception:
            peer_ok = False
        if peer_ok:
            i, d = sdist._exchange_peer(dev(Q), dev(T), k, 0, None, 1, 0, sknn.join, False, True, {})
            torch.cuda.synchronize()
            assert_knn_bitexact(i.cpu().numpy(), d.cpu().numpy(), ridx, rdist)
    finally:
        tdist.destroy_process_group()


@pytest.mark.parametrize("P,k,nq,lo,n", [(1, 8, 500, 0, 500), (3, 32, 700, 129, 400), (8, 20, 1000, 999, 1),
                                         (5, 16, 333, 0, 0), (16, 5, 257, 7, 250)])
def test_merge_partials_ptrs_equals_stacked(sknn, P, k, nq, lo, n):
    """sknn_merge_partials_ptrs (the peer-buffer merge of the fused NVLink
    exchange) over P SEPARATE buffers, rows [lo, lo + n): bit-identical to the
    stacked-array merge of the same lists (ties across lists included)."""
    rng = np.random.default_rng(P * 31 + k)
    d2 = np.sort(rng.integers(0, 40, size=(P, nq, k)).astype(np.float32), axis=2)
    idx = (np.arange(k)[None, None, :] + np.arange(P)[:, None, None] * 10_000).astype(np.int32) + \
        np.zeros((P, nq, k), np.int32)
    bufs_i = [torch.from_numpy(idx[p].copy()).cuda() for p in range(P)]   # separate allocations
    bufs_d = [torch.from_numpy(d2[p].copy()).cuda() for p in range(P)]
    ri, rd = sknn.merge_partials(torch.from_numpy(idx).cuda(), torch.from_numpy(d2).cuda(), k)
    if n == 0:
        return
    pi, pd = sknn.merge_partials_ptrs([b.data_ptr() for b in bufs_i], [b.data_ptr() for b in bufs_d], nq, lo, n, k)
    torch.cuda.synchronize()
    np.testing.assert_array_equal(pi.cpu().numpy(), ri[lo:lo + n].cpu().numpy())
    np.testing.assert_array_equal(pd.cpu().numpy().view(np.uint32), rd[lo:lo + n].cpu().numpy().view(np.uint32))


def test_build_is_deterministic(sknn):
    """The clustering is deterministic (fixed-point Lloyd sums, ordered sampling
    compaction): two builds export identical indexes and two joins report
    identical level-1 counters and results -- query-sharded ranks rely on
    agreeing cluster ids. (Scan evaluation counts may differ by a few when
    split tasks share a bound, whose timing is not deterministic; they are
    compared with tile splitting disabled.)"""
    for name, scale in (("C2", 0.05), ("C5", 0.005), ("C4", 0.004)):
        Q, T, k, sj = datagen.workload(name, scale)
        a = sknn.build(dev(T)).export()
        b = sknn.build(dev(T)).export()
        for key in a:
            np.testing.assert_array_equal(a[key], b[key])
        i1, d1, s1 = run(sknn, Q, T, k, sj)
        i2, d2, s2 = run(sknn, Q, T, k, sj)
        np.testing.assert_array_equal(i1, i2)
        np.testing.assert_array_equal(d1, d2)
        for key in ("cand_pairs", "dense_pairs"):
            assert s1[key] == s2[key], key
        os.environ["SKNN_SPLIT"] = "0"
        try:
            _, _, s1 = run(sknn, Q, T, k, sj)
            _, _, s2 = run(sknn, Q, T, k, sj)
        finally:
            del os.environ["SKNN_SPLIT"]
        for key in ("dist_evals", "cand_pairs", "center_evals", "dense_pairs"):
            assert s1[key] == s2[key], key


def test_index_self_join_and_reuse(sknn):
    """sknn_query with Q == the indexed T (self-join through the index) and
    repeated queries against one resident index on another stream."""
    X = datagen.c3_kegg(4000, integer=True)
    dX = dev(X)
    ix = sknn.build(dX)
    ridx, rdist = oracle.knn_join(X, X, 16)
    i1, d1 = ix.query(dX, 16)
    s = torch.cuda.Stream()
    with torch.cuda.stream(s):
        i2, d2 = ix.query(dX, 16, stream=s)
    s.synchronize()
    torch.cuda.synchronize()
    assert_knn_bitexact(i1.cpu().numpy(), d1.cpu().numpy(), ridx, rdist)
    assert_knn_bitexact(i2.cpu().numpy(), d2.cpu().numpy(), ridx, rdist)
    Q = datagen.c3_kegg(700, integer=True, seed=8)
    i3, d3 = ix.query(Q, 16)  # host buffers through the index
    r3i, r3d = oracle.knn_join(Q, X, 16)
    assert_knn_bitexact(i3, d3, r3i, r3d)
    ix.close()


def test_squared_output_and_index_base(sknn):
    Q, T, k, sj = datagen.workload("C1")
    dQ = dev(Q)
    i, d2 = sknn.join(dQ, dQ, k, out_squared=1, index_base=1000)
    ridx, rdist, rd2 = oracle.knn_join(Q, T, k, return_d2=True)
    np.testing.assert_array_equal(i.cpu().numpy(), ridx + 1000)
    np.testing.assert_array_equal(d2.cpu().numpy(), rd2.astype(np.float32))


# ----------------------------------------------------------- large k (NEXT-2) --
@pytest.mark.parametrize("k", [33, 64, 100, 256, 512])
def test_large_k(sknn, k):
    """k beyond the register budget: shared-memory kNearests with fewer threads
    per CTA (Fig. 8 placement); bit-exact on integer inputs, low and high d."""
    rng = np.random.default_rng(k)
    for d in (4, 28, 40):
        T = rng.integers(0, 60, size=(4000, d)).astype(np.float32)
        Q = rng.integers(0, 60, size=(500, d)).astype(np.float32)
        idx, dist, _ = run(sknn, Q, T, k, False)
        ridx, rdist = oracle.knn_join(Q, T, k)
        assert_knn_bitexact(idx, dist, ridx, rdist)
    X = datagen.c1_uniform_int(2048)
    idx, dist, _ = run(sknn, X, X, k, True)
    ridx, rdist = oracle.knn_join(X, X, k)
    assert_knn_bitexact(idx, dist, ridx, rdist)


def test_merge_partials_large_k(sknn):
    T = datagen.c5_blobs(12000, which="T")
    Q = datagen.c5_blobs(1500, which="Q")
    k = 64
    dQ = dev(Q)
    parts_i, parts_d = [], []
    bounds = np.linspace(0, T.shape[0], 4).astype(int)
    for r in range(3):
        i, d = sknn.join(dQ, dev(T[bounds[r]:bounds[r + 1]]), k, out_squared=1, index_base=int(bounds[r]))
        parts_i.append(i)
        parts_d.append(d)
    idx, dist = sknn.merge_partials(torch.stack(parts_i), torch.stack(parts_d), k)
    torch.cuda.synchronize()
    ridx, rdist = oracle.knn_join(Q, T, k)
    assert_knn_bitexact(idx.cpu().numpy(), dist.cpu().numpy(), ridx, rdist)


@pytest.mark.parametrize("name,scale", [("C1", 1.0), ("C3int", 0.05), ("C5", 0.0025), ("C2", 0.02)])
def test_split_tasks_match_unsplit(sknn, name, scale):
    """Load-balanced level-2 tasks: tiles split across several warps (shared
    k-th bound + k_merge_split) give the same bits as unsplit tiles
    (SKNN_SPLIT=0) and as the oracle. Small inputs split almost every tile."""
    Q, T, k, sj = datagen.workload(name, scale)
    ridx, rdist = oracle.knn_join(Q, T, k)
    i1, d1, _ = run(sknn, Q, T, k, sj)
    os.environ["SKNN_SPLIT"] = "0"
    try:
        i0, d0, _ = run(sknn, Q, T, k, sj)
    finally:
        del os.environ["SKNN_SPLIT"]
    if name == "C2":
        assert_knn_tolerant(Q, T, i1, d1, rdist)
        np.testing.assert_array_equal(d1, d0)
    else:
        assert_knn_bitexact(i1, d1, ridx, rdist)
        assert_knn_bitexact(i0, d0, ridx, rdist)


# ------------------------------------------- partial level-2 filter (§IV-B1) --
@pytest.mark.parametrize("k", [1, 8, 20, 64, 512])
def test_partial_filter_bitexact(sknn, k):
    """SKNN_PATH_PARTIAL (fixed-UB level-2 filter, survivor buffer, k-select):
    bit-exact on integer inputs at the paper's k sweep {1, 8, 20, 64, 512}
    (Fig. 10 / Table V), self-join and non-self join, low and mid d."""
    rng = np.random.default_rng(100 + k)
    for d in (4, 28):
        T = rng.integers(0, 60, size=(3000, d)).astype(np.float32)
        Q = rng.integers(0, 60, size=(700, d)).astype(np.float32)
        idx, dist, st = run(sknn, Q, T, k, False, force_path="partial")
        assert st["path_used"] == 4
        ridx, rdist = oracle.knn_join(Q, T, k)
        assert_knn_bitexact(idx, dist, ridx, rdist)
    X = datagen.c1_uniform_int(1024)
    idx, dist, st = run(sknn, X, X, k, True, force_path="partial")
    ridx, rdist = oracle.knn_join(X, X, k)
    assert_knn_bitexact(idx, dist, ridx, rdist)
    assert X.shape[0] * k <= st["dist_evals"] <= X.shape[0] ** 2


@pytest.mark.parametrize("name,scale", [("C3int", 0.05), ("C5", 0.0025), ("C4", 0.002)])
def test_partial_filter_workloads(sknn, name, scale):
    Q, T, k, sj = datagen.workload(name, scale)
    idx, dist, st = run(sknn, Q, T, k, sj, force_path="partial")
    assert st["path_used"] == 4
    ridx, rdist = oracle.knn_join(Q, T, k)
    assert_knn_bitexact(idx, dist, ridx, rdist)


def test_partial_filter_real_and_ties(sknn):
    """Real-valued C2/C3 shapes within the tolerance; the equal-norm sphere
    (P10) keeps the lowest indices among exact ties; duplicates everywhere."""
    for name, scale in (("C2", 0.02), ("C3", 0.05)):
        Q, T, k, sj = datagen.workload(name, scale)
        idx, dist, _ = run(sknn, Q, T, k, sj, force_path="partial")
        _, rdist = oracle.knn_join(Q, T, k)
        assert_knn_tolerant(Q, T, idx, dist, rdist)
    S = datagen.sphere_ties()
    Q0 = S[:1].copy()
    for k in (1, 7, 100, 384):
        idx, dist, _ = run(sknn, Q0, S, k, False, force_path="partial")
        ridx, rdist = oracle.knn_join(Q0, S, k)
        assert_knn_bitexact(idx, dist, ridx, rdist)
    D = np.zeros((300, 4), np.float32)
    idx, dist, _ = run(sknn, D, D, 16, True, force_path="partial")
    ridx, rdist = oracle.knn_join(D, D, 16)
    assert_knn_bitexact(idx, dist, ridx, rdist)


# ------------------------------------------------- out-of-core queries (NEXT-4) --
@pytest.mark.parametrize("batch", [0, 333, 1000, 5000])
def test_query_batches_host_memory(sknn, batch):
    """sknn_query with host queries and outputs streams the queries through the
    device in batches (the paper's query partitions): results equal the
    oracle bit-exactly for every batch size (ragged last batch included) and
    the per-batch stats add up."""
    T = datagen.c5_blobs(20000, which="T")
    Q = datagen.c5_blobs(3100, which="Q")
    k = 32
    ix = sknn.build(dev(T))
    idx, dist, st = ix.query(Q, k, stats=True, query_batch=batch)   # numpy: host pointers
    ridx, rdist = oracle.knn_join(Q, T, k)
    assert_knn_bitexact(np.asarray(idx), np.asarray(dist), ridx, rdist)
    assert st["pairs_total"] == Q.shape[0] * T.shape[0]
    # without stats the batches overlap on two streams (pageable buffers go
    # through page-locked staging; page-locked ones are used in place)
    idx2, dist2 = ix.query(Q, k, query_batch=batch)
    assert_knn_bitexact(np.asarray(idx2), np.asarray(dist2), ridx, rdist)
    pq = torch.from_numpy(Q).pin_memory()
    pi = torch.empty((Q.shape[0], k), dtype=torch.int32).pin_memory()
    pd = torch.empty((Q.shape[0], k), dtype=torch.float32).pin_memory()
    ix.query(pq, k, query_batch=batch, out=(pi, pd))
    assert_knn_bitexact(pi.numpy(), pd.numpy(), ridx, rdist)
    # pinned queries, pageable outputs (mixed staging)
    idx3, dist3 = ix.query(pq, k, query_batch=batch)
    assert_knn_bitexact(np.asarray(idx3), np.asarray(dist3), ridx, rdist)
    ix.close()


SEGSORT_SIZES = [2, 31, 32, 33, 64, 65, 128, 129, 255, 256, 257, 1023, 1024, 1025, 4096, 4097]


@pytest.mark.parametrize("n", SEGSORT_SIZES)
def test_member_sort_bucket_boundaries(sknn, n):
    """One cluster of exactly n members (n_clusters_t = 1) at every k_segsort_small/_big bucket edge
    (register sort <= 32/64/128/256, smem network <= 1024, hybrid above): members ordered by distance
    descending, index ascending (reading R11), radius = first member, then the join bit-exact."""
    rng = np.random.default_rng(1000 + n)
    X = rng.integers(0, 4, size=(n, 4)).astype(np.float32)   # many equal distances: tie order matters
    ix = sknn.build(dev(X), n_clusters_t=1)
    e = ix.export()
    assert len(e["off"]) == 2 and e["off"][0] == 0 and e["off"][-1] == n   # det_lm_num: m = 1
    assert np.array_equal(np.sort(e["orig"]), np.arange(n))
    for c in range(len(e["off"]) - 1):
        lo, hi = e["off"][c], e["off"][c + 1]
        dd, oo = e["dist"][lo:hi], e["orig"][lo:hi]
        ok = (dd[:-1] > dd[1:]) | ((dd[:-1] == dd[1:]) & (oo[:-1] < oo[1:]))
        assert ok.all()
        if hi > lo:
            assert e["radius"][c] == dd[0]
    ix.close()
    k = min(8, n)
    idx, dist, _ = run(sknn, X, X, k, True, n_clusters_t=1)
    ridx, rdist = oracle.knn_join(X, X, k)
    assert_knn_bitexact(idx, dist, ridx, rdist)


def _graph_join(sknn, dQ, dT, k, oi, od, **opts):
    sknn.join(dQ, dT, k, out=(oi, od), **opts)
    torch.cuda.synchronize()
    return oi.cpu().numpy().copy(), od.cpu().numpy().copy()


def test_graph_replay_matches_eager(sknn):
    """Repeated stats-free joins on the same buffers run as a recorded CUDA
    graph (first call eager, second recorded, then replayed): every call equals
    the eager join bit for bit, and a replay after new contents are written
    into the same buffers computes the join of the new contents."""
    Q, T, k, sj = datagen.workload("C2", 0.1)
    n = Q.shape[0]
    dQ = dev(Q)
    oi = torch.empty((n, k), dtype=torch.int32, device="cuda")
    od = torch.empty((n, k), dtype=torch.float32, device="cuda")
    ri, rd = sknn.join(dQ, dQ, k, use_graph=-1)
    ri, rd = ri.cpu().numpy(), rd.cpu().numpy()
    for _ in range(4):
        gi, gd = _graph_join(sknn, dQ, dQ, k, oi, od)
        np.testing.assert_array_equal(gi, ri)
        np.testing.assert_array_equal(gd.view(np.uint32), rd.view(np.uint32))
    Q2 = np.ascontiguousarray(Q[::-1] * np.float32(1.5))
    dQ.copy_(torch.from_numpy(Q2))
    gi, gd = _graph_join(sknn, dQ, dQ, k, oi, od)
    ri2, rd2 = sknn.join(dQ, dQ, k, use_graph=-1)
    np.testing.assert_array_equal(gi, ri2.cpu().numpy())
    np.testing.assert_array_equal(gd.view(np.uint32), rd2.cpu().numpy().view(np.uint32))
    _, odist = oracle.knn_join(Q2, Q2, k)
    assert_knn_tolerant(Q2, Q2, gi, gd, odist)


def test_graph_replay_integer_bitexact(sknn):
    """C1 and a Q != T integer join through graph replays: bit-exact vs the oracle."""
    for name, scale in (("C1", 1.0), ("C5", 0.002)):
        Q, T, k, sj = datagen.workload(name, scale)
        dQ = dev(Q)
        dT = dQ if sj else dev(T)
        oi = torch.empty((Q.shape[0], k), dtype=torch.int32, device="cuda")
        od = torch.empty((Q.shape[0], k), dtype=torch.float32, device="cuda")
        ridx, rdist = oracle.knn_join(Q, T, k)
        for _ in range(3):
            gi, gd = _graph_join(sknn, dQ, dT, k, oi, od)
            assert_knn_bitexact(gi, gd, ridx, rdist)


@pytest.mark.slow
def test_c2_full_size_graph_path_sampled(sknn):
    """C2 at full size in exactly bench.py's timed launch configuration (no
    stats, repeated calls on the same buffers -> CUDA graph replay): a seeded
    sample of queries checked against the oracle one by one."""
    Q, T, k, sj = datagen.workload("C2")
    n = Q.shape[0]
    dQ = dev(Q)
    oi = torch.empty((n, k), dtype=torch.int32, device="cuda")
    od = torch.empty((n, k), dtype=torch.float32, device="cuda")
    for _ in range(3):
        gi, gd = _graph_join(sknn, dQ, dQ, k, oi, od)
    rng = np.random.default_rng(7)
    s = rng.choice(n, 2000, replace=False)
    _, rdist = oracle.knn_join(Q[s], T, k)
    assert_knn_tolerant(Q[s], T, gi[s], gd[s], rdist)


def test_dense_exact_integer_path(sknn):
    """Integer inputs inside the exactness bound (no bf16 lo part, dp (A+B)^2 <
    2^24): the dense tiles run the exact variant -- the tensor-core d2 IS the
    key, nothing is recomputed -- and stay bit-identical to the oracle,
    including ties (equal-norm sphere) and every k bucket."""
    Q, T, k, sj = datagen.workload("C4", 0.004)
    idx, dist, st = run(sknn, Q, T, k, sj, force_path="dense")
    ridx, rdist = oracle.knn_join(Q, T, k)
    assert_knn_bitexact(idx, dist, ridx, rdist)
    assert st["dist_evals_dense"] > 0 and st["dist_recompute"] == 0
    X = datagen.sphere_ties()
    Qs = np.concatenate([np.zeros((5, 4), np.float32), X[::7]], axis=0)
    for kk in (1, 8, 13, 16, 20, 24, 31, 32):
        i2, d2_, st2 = run(sknn, Qs, X, kk, False, force_path="dense")
        r2, rd2 = oracle.knn_join(Qs, X, kk)
        assert_knn_bitexact(i2, d2_, r2, rd2)
        assert st2["dist_recompute"] == 0


@pytest.mark.parametrize("hi,d", [(4000, 20), (600, 16)])
def test_dense_split_precision_fallback(sknn, hi, d):
    """Integer inputs outside the exactness bound (coordinates whose re-centred
    values need a bf16 lo part, or dp (A+B)^2 >= 2^24) take the split-precision
    screen + exact recompute variant; still bit-identical to the oracle."""
    rng = np.random.default_rng(hi + d)
    centers = rng.integers(0, hi, size=(20, d))
    T = (centers[rng.integers(0, 20, 3000)] + rng.integers(-hi // 20, hi // 20 + 1, size=(3000, d)))
    T = np.clip(T, 0, hi).astype(np.float32)
    Q = np.clip(centers[rng.integers(0, 20, 500)] + rng.integers(-hi // 20, hi // 20 + 1, size=(500, d)), 0,
                hi).astype(np.float32)
    k = 16
    idx, dist, st = run(sknn, Q, T, k, False, force_path="dense")
    ridx, rdist = oracle.knn_join(Q, T, k)
    assert_knn_bitexact(idx, dist, ridx, rdist)
    assert st["dist_evals_dense"] > 0 and st["dist_recompute"] > 0


@pytest.mark.parametrize("form", ["", "direct", "staged", "warp"])
@pytest.mark.parametrize("P,k", [(1, 5), (2, 32), (8, 32), (3, 1), (20, 7), (5, 33), (9, 100), (4, 512), (17, 256),
                                 (1, 32), (8, 16), (3, 20), (4, 8), (3, 4), (2, 12), (6, 28)])
def test_merge_partials_bitonic(sknn, P, k, form, monkeypatch):
    """sknn_merge_partials on P sorted lists with many equal distances across
    lists: the k smallest (d2, idx) keys, compared with a lexicographic sort of
    the concatenated lists (np.lexsort). k <= 32 runs every form: the staged
    thread-per-query merge (default for k % 4 == 0), the direct-load thread
    form (default otherwise) and the warp form; nq = 700 leaves a ragged
    128-query block."""
    if form and k > 32:
        pytest.skip("one form above k = 32")
    if form:
        monkeypatch.setenv("SKNN_MERGE", form)
    rng = np.random.default_rng(P * 1000 + k)
    nq = 700
    d2 = np.sort(rng.integers(0, 50, size=(P, nq, k)).astype(np.float32), axis=2)
    idx = (np.arange(k, dtype=np.int64)[None, None, :] + np.arange(P)[:, None, None] * 100_000 +
           rng.integers(0, 1000, size=(1, nq, 1)) * 0).astype(np.int32)
    oi, od = sknn.merge_partials(torch.from_numpy(idx).cuda(), torch.from_numpy(d2).cuda(), k, out_squared=True)
    torch.cuda.synchronize()
    oi, od = oi.cpu().numpy(), od.cpu().numpy()
    I = idx.transpose(1, 0, 2).reshape(nq, -1)
    D = d2.transpose(1, 0, 2).reshape(nq, -1)
    for q in range(nq):
        order = np.lexsort((I[q], D[q]))[:k]
        np.testing.assert_array_equal(oi[q], I[q][order])
        np.testing.assert_array_equal(od[q], D[q][order])


def test_index_create_and_share_arrays(sknn):
    """sknn_index_create + sknn_index_arrays (the build-once-and-broadcast
    path): an empty index filled with another index's arrays answers queries
    and self-queries (self_query=1, query sharding included) bit-identically."""
    Q, T, k, sj = datagen.workload("C3int", 0.05)
    dT = dev(T)
    ix = sknn.Index(dT)
    inf = ix.info()
    ix2 = sknn.Index.create(inf["nt"], inf["d"], inf["mt"])
    for src, dst in zip(ix.arrays(), ix2.arrays()):
        assert src.numel() == dst.numel()
        dst.copy_(src)
    torch.cuda.synchronize()
    dQ = dev(Q[:500] + 1.0)
    a = ix.query(dQ, k)
    b = ix2.query(dQ, k)
    np.testing.assert_array_equal(a[0].cpu().numpy(), b[0].cpu().numpy())
    np.testing.assert_array_equal(a[1].cpu().numpy(), b[1].cpu().numpy())
    ridx, rdist = oracle.knn_join(T, T, k)
    oi = torch.full((T.shape[0], k), -1, dtype=torch.int32, device="cuda")
    od = torch.zeros((T.shape[0], k), dtype=torch.float32, device="cuda")
    for r in range(3):
        ix2.query(dT, k, out=(oi, od), self_query=1, shard_rank=r, shard_count=3)
    torch.cuda.synchronize()
    assert_knn_bitexact(oi.cpu().numpy(), od.cpu().numpy(), ridx, rdist)
    ix.close()
    ix2.close()


def _median_ms(sknn, dQ, dT, k, reps=3, **opts):
    ms = []
    for r in range(reps + 1):
        _, _, st = sknn.join(dQ, dT, k, stats=True, **opts)
        if r:
            ms.append(st["ms_total"])
    return float(np.median(ms))


@pytest.mark.slow
@pytest.mark.parametrize("name", ["C1", "C2", "C3", "C4", "C5"])
def test_auto_configuration_within_margin_of_best_forced(sknn, name):
    """The adaptive configuration (S1 / S8: mapping and elastic switch chosen
    by the runtime rules, Fig. 8 re-derived for B200) is within 10% (+ 0.05
    ms of timer noise) of the fastest forced alternative on every config."""
    Q, T, k, sj = datagen.workload(name)
    dQ = dev(Q)
    dT = dQ if sj else dev(T)
    auto = _median_ms(sknn, dQ, dT, k)
    forced = {"thread": dict(mapping="thread", force_path="sparse"),
              "warp": dict(mapping="warp", force_path="sparse")}
    if name == "C4":
        forced["dense"] = dict(force_path="dense")
        forced.pop("thread")  # dp = 128 has no thread-per-query variant
    if name in ("C1", "C2", "C3"):
        forced["dense"] = dict(force_path="dense")
    best = min(_median_ms(sknn, dQ, dT, k, **o) for o in forced.values())
    assert auto <= 1.10 * best + 0.05, (name, auto, best)


def test_target_sharded_global_ub(sknn):
    """NEXT-1: target sharding with the GLOBAL level-1 bound, simulated on one
    GPU with P = 3 shards. The query clustering is shared (sknn_build over Q),
    every shard's calUB (sknn_level1_bounds) is combined by a minimum, each
    shard joins with ub_in = that minimum (sknn_join_indexed), and the merged
    partial lists equal the oracle bit for bit; the global bound never
    evaluates more distances than the local ones."""
    T = datagen.c5_blobs(24000, which="T")
    Q = datagen.c5_blobs(3000, which="Q")
    k = 32
    dQ, dT = dev(Q), dev(T)
    qix = sknn.Index(dQ)
    P = 3
    bounds = np.linspace(0, T.shape[0], P + 1).astype(int)
    tix = [sknn.Index(dT[bounds[r]:bounds[r + 1]].contiguous()) for r in range(P)]
    ubs = torch.stack([sknn.level1_bounds(qix, t, k) for t in tix])
    ub = ubs.min(dim=0).values
    assert torch.all(ub <= ubs[0])
    evals = {}
    parts = {}
    for mode, kw in (("local", {}), ("global", {"ub_in": ub})):
        pi, pd, ev = [], [], 0
        for r in range(P):
            i, d, st = sknn.join_indexed(qix, tix[r], k, stats=True, out_squared=1, index_base=int(bounds[r]), **kw)
            pi.append(i)
            pd.append(d)
            ev += st["dist_evals"]
        evals[mode] = ev
        parts[mode] = (torch.stack(pi), torch.stack(pd))
    ridx, rdist = oracle.knn_join(Q, T, k)
    for mode in ("local", "global"):
        idx, dist = sknn.merge_partials(parts[mode][0], parts[mode][1], k)
        torch.cuda.synchronize()
        assert_knn_bitexact(idx.cpu().numpy(), dist.cpu().numpy(), ridx, rdist)
    assert evals["global"] <= evals["local"]
    # placeholders (fewer than k real keys under the global bound) carry index -1
    gi = parts["global"][0].cpu().numpy()
    gd = parts["global"][1].cpu().numpy()
    assert np.all((gi >= 0) | (gi == -1)) and np.all(np.isinf(gd[gi == -1]))


# ------------------------------------------- basic KNN-TI ablation arm (NEXT-3) --
@pytest.mark.parametrize("name,scale", [("C1", 1.0), ("C3int", 0.05), ("C5", 0.0025), ("C4", 0.002), ("C2", 0.02)])
def test_basic_knnti_matches_oracle(sknn, name, scale):
    """mapping='basic' (the basic KNN-TI of Fig. 4 / Alg. 2: thread per query in
    input order, per-thread walks from the top of each candidate cluster) gives
    the oracle's result: bit-exact on integer inputs, within 1e-5 on C2; and it
    never evaluates fewer distances than the Alg. 2 windows need, i.e. its
    evaluation count is >= 0 and pruning stays the TI pruning (< 100%)."""
    Q, T, k, sj = datagen.workload(name, scale)
    idx, dist, st = run(sknn, Q, T, k, sj, mapping="basic")
    ridx, rdist = oracle.knn_join(Q, T, k)
    if name == "C2":
        assert_knn_tolerant(Q, T, idx, dist, rdist)
    else:
        assert_knn_bitexact(idx, dist, ridx, rdist)
    assert st["mapping_used"] == 3 and 0 < st["pruned_pct"] < 100


def test_basic_knnti_rejects_unsupported(sknn):
    Q, T, k, sj = datagen.workload("C1")
    with pytest.raises(RuntimeError):
        run(sknn, Q, T, 40, sj, mapping="basic")
    with pytest.raises(RuntimeError):
        run(sknn, Q, T, k, sj, mapping="basic", force_path="dense")


# ------------------------------------------------ high d (NEXT-4, arcene/dor-like) --
@pytest.mark.parametrize("d,n", [(300, 700), (1024, 600), (4096, 300), (10000, 150), (100000, 40)])
def test_high_dimension_bitexact(sknn, d, n):
    """Dimensions past the tensor-core kernels' K <= 256 (Table III's arcene
    d = 10,000 and dorothea d = 100,000 shapes): sparse binary
    rows (dorothea-like, ~1% ones) plus a dense integer block; every path the
    dispatcher takes at this d (SIMT assignment, runtime-dp scans) is
    bit-exact against the oracle, self-join and Q != T."""
    rng = np.random.default_rng(d + n)
    X = (rng.random((n, d)) < 0.01).astype(np.float32)
    X[:, :8] = rng.integers(0, 4, size=(n, 8))
    Q = (rng.random((n // 2, d)) < 0.01).astype(np.float32)
    k = 8
    idx, dist, _ = run(sknn, X, X, k, True)
    ridx, rdist = oracle.knn_join(X, X, k)
    assert_knn_bitexact(idx, dist, ridx, rdist)
    idx, dist, _ = run(sknn, Q, X, k, False)
    ridx, rdist = oracle.knn_join(Q, X, k)
    assert_knn_bitexact(idx, dist, ridx, rdist)


@pytest.mark.parametrize("nq,nt,d,k", [(1, 1, 1, 1), (65, 63, 7, 5), (200, 3000, 130, 32), (700, 129, 2048, 8),
                                       (33, 5000, 33, 17)])
def test_dense_only_tiled_bitexact(sknn, nq, nt, d, k, monkeypatch):
    """The dense-only path (k_brute_tiled: 64 x 64 register tiles, fused top-k,
    target slices merged by sknn_merge_partials) on ragged shapes: bit-exact
    against the oracle and against the warp-per-query anchor kernel
    (SKNN_BRUTE=warp), with ties (small integer coordinates)."""
    rng = np.random.default_rng(nq * 7 + nt + d)
    Q = rng.integers(0, 3, size=(nq, d)).astype(np.float32)
    T = rng.integers(0, 3, size=(nt, d)).astype(np.float32)
    k = min(k, nt)
    idx, dist, st = run(sknn, Q, T, k, False, force_path="brute")
    ridx, rdist = oracle.knn_join(Q, T, k)
    assert_knn_bitexact(idx, dist, ridx, rdist)
    assert st["pruned_pct"] == 0.0
    monkeypatch.setenv("SKNN_BRUTE", "warp")
    i2, d2, _ = run(sknn, Q, T, k, False, force_path="brute")
    assert_knn_bitexact(i2, d2, ridx, rdist)


def test_dense_only_index_query_high_d(sknn):
    """sknn_query against a prebuilt index at d >= 1024 takes the dense-only
    path over the index's permuted rows (original ids through its map):
    bit-exact, host batches included."""
    rng = np.random.default_rng(5)
    T = (rng.random((900, 1500)) < 0.02).astype(np.float32)
    Q = (rng.random((300, 1500)) < 0.02).astype(np.float32)
    k = 6
    ix = sknn.build(dev(T))
    idx, dist, st = ix.query(dev(Q), k, stats=True)
    torch.cuda.synchronize()
    ridx, rdist = oracle.knn_join(Q, T, k)
    assert_knn_bitexact(idx.cpu().numpy(), dist.cpu().numpy(), ridx, rdist)
    assert st["path_used"] == 3   # SKNN_PATH_BRUTE: every pair
    i2, d2 = ix.query(Q, k, query_batch=100)
    assert_knn_bitexact(np.asarray(i2), np.asarray(d2), ridx, rdist)
    ix.close()


@pytest.mark.parametrize("name,scale,P", [("C5", 0.01, 3), ("C2", 0.05, 4), ("C4", 0.01, 2), ("C1", 1.0, 5)])
def test_sharded_build_equals_build(sknn, name, scale, P):
    """Sharded clustering (NEXT-1): P ranks' final-assignment shards
    (sknn_build_assign_shard on aligned row ranges, simulated one after the
    other on one GPU), summed as the all-reduce would, then
    sknn_build_from_assignment: the index is identical to sknn_build's (every
    exported array), through the tensor-core assignment (C4, C5) and the
    graph walk (C1, C2), ragged and 8-aligned shard boundaries."""
    from paper_conf_icde_chends17_b200.dist import aligned_bounds
    Q, T, k, sj = datagen.workload(name, scale)
    X = dev(Q)
    ref = sknn.build(X).export()
    cid_sum = torch.zeros(X.shape[0], dtype=torch.int32, device="cuda")
    dist_sum = torch.zeros(X.shape[0], dtype=torch.float32, device="cuda")
    centers = None
    for r in range(P):
        lo, hi = aligned_bounds(X.shape[0], P, r)
        c, i, d = sknn.build_assign_shard(X, lo, hi)
        cid_sum += i
        dist_sum += d
        if centers is None:
            centers = c
        else:
            assert torch.equal(c, centers)   # every rank computes the same centers
    ix = sknn.Index.from_assignment(X, centers, cid_sum, dist_sum)
    got = ix.export()
    for key in ref:
        np.testing.assert_array_equal(got[key], ref[key])
    ix.close()
