"""Multi-process (world_size 2, gloo, CPU) tests of the multi-GPU orchestration
in paper_conf_icde_chends17_b200/dist.py: shard bounds, query-sharded result
assembly, target-sharded partial-list exchange with global indices and the
exact merge. The per-rank join is injected (the CPU oracle restricted to the
rank's shard) and so is the merge (a host reference), because the CUDA
library needs a GPU; the same orchestration code runs with NCCL on B200s.
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import datagen
import oracle


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def oracle_local_join(Q, T, k, out=None, out_squared=0, index_base=0, shard_rank=0, shard_count=1, **_):
    """CPU stand-in for sknn.join with the same calling convention (tests only)."""
    Qn, Tn = Q.numpy(), T.numpy()
    idx, dist_, d2 = oracle.knn_join(Qn, Tn, k, return_d2=True)
    vals = d2.astype(np.float32) if out_squared else dist_
    idx = idx + index_base
    if out is not None:
        # query sharding of a self-join: rows of this rank's "clusters" (here: i % count)
        rows = np.arange(Qn.shape[0]) % shard_count == shard_rank
        out[0][torch.from_numpy(rows)] = torch.from_numpy(idx[rows].astype(np.int32))
        out[1][torch.from_numpy(rows)] = torch.from_numpy(vals[rows])
        return out
    return torch.from_numpy(idx.astype(np.int32)), torch.from_numpy(vals)


def host_merge(all_i, all_d, k, out_squared=False):
    P, nq, _ = all_d.shape
    I = all_i.numpy().transpose(1, 0, 2).reshape(nq, -1)
    D = all_d.numpy().transpose(1, 0, 2).reshape(nq, -1)
    oi = np.empty((nq, k), np.int32)
    od = np.empty((nq, k), np.float32)
    for q in range(nq):
        order = np.lexsort((I[q], D[q]))[:k]
        oi[q] = I[q][order]
        od[q] = D[q][order] if out_squared else np.sqrt(D[q][order].astype(np.float64)).astype(np.float32)
    return torch.from_numpy(oi), torch.from_numpy(od)


def _worker(rank, world, port, results):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    from paper_conf_icde_chends17_b200 import dist as sdist
    try:
        X = datagen.c1_uniform_int(600)
        Q = datagen.c1_uniform_int(150, seed=9)
        k = 8
        # target sharding
        lo, hi = sdist.shard_bounds(X.shape[0], world, rank)
        i, d = sdist.join_target_sharded(torch.from_numpy(Q), torch.from_numpy(X[lo:hi]).contiguous(), k, lo,
                                         local_join=oracle_local_join, merge=host_merge)
        # target sharding, all-to-all exchange (NEXT-1): a ragged query count
        Q2 = datagen.c1_uniform_int(151, seed=10)
        ai, ad = sdist.join_target_sharded(torch.from_numpy(Q2), torch.from_numpy(X[lo:hi]).contiguous(), k, lo,
                                           local_join=oracle_local_join, merge=host_merge, exchange="all_to_all")
        si_, sd_ = sdist.join_target_sharded(torch.from_numpy(Q2), torch.from_numpy(X[lo:hi]).contiguous(), k, lo,
                                             local_join=oracle_local_join, merge=host_merge, exchange="all_to_all",
                                             gather=False)
        # all-to-all with the exchange pruned by the min-over-ranks k-th distance (NEXT-1)
        pst = {}
        pi_, pd_ = sdist.join_target_sharded(torch.from_numpy(Q2), torch.from_numpy(X[lo:hi]).contiguous(), k, lo,
                                             local_join=oracle_local_join, merge=host_merge, exchange="all_to_all",
                                             prune=True, stats=pst)
        # sharded clustering (NEXT-1): each rank assigns its aligned rows, one all-reduce
        # SUM per array assembles the assignment (CPU stand-in for the assignment)
        def fake_assign(Xs, lo_, hi_, **_):
            C = Xs[:4].clone()
            d2 = ((Xs[:, None, :] - C[None]) ** 2).sum(-1)
            ci = torch.zeros(Xs.shape[0], dtype=torch.int32)
            di = torch.zeros(Xs.shape[0], dtype=torch.float32)
            ci[lo_:hi_] = d2.argmin(1).int()[lo_:hi_]
            di[lo_:hi_] = d2.min(1).values.sqrt()[lo_:hi_]
            return C, ci, di
        bi_, bd_ = sdist.build_index_sharded(torch.from_numpy(X), assign_shard=fake_assign,
                                             from_assignment=lambda X_, c, i_, d_, **o: (i_.clone(), d_.clone()))
        # query sharding, non-self join: interleaved query clusters (default) and contiguous rows
        qi, qd = sdist.join_query_sharded(torch.from_numpy(Q), torch.from_numpy(X), k, self_join=False,
                                          local_join=oracle_local_join)
        wi, wd = sdist.join_query_sharded(torch.from_numpy(Q), torch.from_numpy(X), k, self_join=False,
                                          local_join=oracle_local_join, partition="rows")
        # query sharding, self join (cluster-interleaved rows, assembled by all-reduce)
        Xt = torch.from_numpy(X)
        si, sd = sdist.join_query_sharded(Xt, Xt, k, local_join=oracle_local_join)
        results[rank] = (i.numpy(), d.numpy(), qi.numpy(), qd.numpy(), si.numpy(), sd.numpy(),
                         ai.numpy(), ad.numpy(), si_.numpy(), sd_.numpy(), wi.numpy(), wd.numpy(),
                         pi_.numpy(), pd_.numpy(), pst["entries_sent"], pst["entries_unpruned"],
                         bi_.numpy(), bd_.numpy())
    finally:
        dist.destroy_process_group()


def test_shard_bounds():
    from paper_conf_icde_chends17_b200.dist import shard_bounds
    for n in (0, 1, 7, 100, 101):
        for w in (1, 2, 3, 8):
            parts = [shard_bounds(n, w, r) for r in range(w)]
            assert parts[0][0] == 0 and parts[-1][1] == n
            assert all(parts[r][1] == parts[r + 1][0] for r in range(w - 1))
            sizes = [b - a for a, b in parts]
            assert max(sizes) - min(sizes) <= 1


def test_two_rank_gloo_matches_single_join():
    world = 2
    port = _free_port()
    mgr = mp.Manager()
    results = mgr.dict()
    mp.spawn(_worker, args=(world, port, results), nprocs=world, join=True)
    X = datagen.c1_uniform_int(600)
    Q = datagen.c1_uniform_int(150, seed=9)
    k = 8
    ridx, rdist = oracle.knn_join(Q, X, k)
    sidx, sdist_ = oracle.knn_join(X, X, k)
    Q2 = datagen.c1_uniform_int(151, seed=10)
    aidx, adist = oracle.knn_join(Q2, X, k)
    from paper_conf_icde_chends17_b200.dist import shard_bounds
    for r in range(world):
        i, d, qi, qd, si, sd, ai, ad, ri, rd, wi, wd, pi_, pd_, sent, unpruned, bi_, bd_ = results[r]
        Xt_ = torch.from_numpy(X)
        d2_ = ((Xt_[:, None, :] - Xt_[:4][None]) ** 2).sum(-1)
        np.testing.assert_array_equal(bi_, d2_.argmin(1).int().numpy())   # sharded assignment, assembled
        np.testing.assert_array_equal(bd_, d2_.min(1).values.sqrt().numpy())
        np.testing.assert_array_equal(pi_, aidx)     # pruned all-to-all exchange, assembled: exact
        np.testing.assert_array_equal(pd_, adist)
        assert sent < unpruned                        # entries above the min k-th never travel
        np.testing.assert_array_equal(wi, ridx)      # query-sharded by row slices, assembled
        np.testing.assert_array_equal(wd, rdist)
        np.testing.assert_array_equal(ai, aidx)      # all-to-all exchange, assembled
        np.testing.assert_array_equal(ad, adist)
        lo, hi = shard_bounds(Q2.shape[0], world, r)
        np.testing.assert_array_equal(ri, aidx[lo:hi])  # all-to-all, this rank's merged slice
        np.testing.assert_array_equal(rd, adist[lo:hi])
        np.testing.assert_array_equal(i, ridx)       # target-sharded == single join (bit-exact)
        np.testing.assert_array_equal(d, rdist)
        np.testing.assert_array_equal(qi, ridx)      # query-sharded, assembled
        np.testing.assert_array_equal(qd, rdist)
        np.testing.assert_array_equal(si, sidx)      # self-join, cluster-interleaved shards
        np.testing.assert_array_equal(sd, sdist_)


class _FakeIndex:
    """CPU stand-in for sknn.Index with the same build/create/info/arrays
    surface (the orchestration of build_index_broadcast is what is tested)."""

    def __init__(self, arrays, nt, d, mt):
        self._arr, self.nt, self.d, self.mt = arrays, nt, d, mt

    def info(self):
        return dict(nt=self.nt, d=self.d, mt=self.mt)

    def arrays(self):
        return self._arr


def _fake_build(X, **_):
    n, d = X.shape
    mt = 7
    g = torch.Generator().manual_seed(5)
    arrs = [torch.randint(0, 255, (nb,), dtype=torch.uint8, generator=g)
            for nb in (n * d * 4, n * 4, n * 4, (mt + 1) * 4, mt * d * 4, mt * 4, mt * 16)]
    return _FakeIndex(arrs, n, d, mt)


def _fake_create(nt, d, mt, **_):
    arrs = [torch.zeros(nb, dtype=torch.uint8) for nb in (nt * d * 4, nt * 4, nt * 4, (mt + 1) * 4, mt * d * 4,
                                                         mt * 4, mt * 16)]
    return _FakeIndex(arrs, nt, d, mt)


def _bcast_worker(rank, world, port, results):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    from paper_conf_icde_chends17_b200 import dist as sdist
    try:
        X = torch.from_numpy(datagen.c1_uniform_int(50))
        ix = sdist.build_index_broadcast(X, build=_fake_build, create=_fake_create)
        results[rank] = (ix.info(), [a.numpy().copy() for a in ix.arrays()])
    finally:
        dist.destroy_process_group()


def test_build_index_broadcast_two_ranks():
    """Build once on rank 0, broadcast the index geometry and every array:
    rank 1 ends with an identical index (the query-sharded mode's alternative
    to replicated builds)."""
    world = 2
    port = _free_port()
    mgr = mp.Manager()
    results = mgr.dict()
    mp.spawn(_bcast_worker, args=(world, port, results), nprocs=world, join=True)
    i0, a0 = results[0]
    i1, a1 = results[1]
    assert i0 == i1 == dict(nt=50, d=4, mt=7)
    assert len(a0) == len(a1) == 7
    for x, y in zip(a0, a1):
        np.testing.assert_array_equal(x, y)
