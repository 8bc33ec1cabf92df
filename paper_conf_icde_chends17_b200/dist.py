"""Multi-GPU KNN join over torch.distributed (one process per GPU, NCCL).

SURVEY.md §8(e). Two modes:

* Query sharding (default; north_star "sharding queries, with the target
  index and cluster metadata replicated"): every rank holds all of T. For a
  self-join every rank clusters T identically (seeded, deterministic sizes)
  and processes the query clusters c with c % P == rank
  (``sknn_options.shard_rank/shard_count``); a Q != T join does the same over
  the clustering of all of Q (``partition="clusters"``, default) or takes the
  contiguous query rows [r*nq/P, (r+1)*nq/P) (``partition="rows"``). No
  data-path collective; the optional result assembly is one collective outside
  the join (one all-reduce of packed (dist, idx) keys, or an all-gather of the
  row slices).
* Target sharding: rank r owns T[r*nt/P, (r+1)*nt/P), computes partial k-lists
  of ALL queries with squared distances and global indices (``out_squared``,
  ``index_base``), the partial lists are exchanged with one all-gather over
  NVLink and merged exactly by ``sknn_merge_partials`` (the paper's merge of
  sorted per-thread heaps, across ranks). The (d2, index) keys are
  global and the merge is a selection on their total order, so the result is
  bit-identical to the single-GPU join. ``exchange="all_to_all"`` (SURVEY
  §8(f) NEXT-1) instead sends each rank only the partial lists of ITS query
  rows [r*nq/P, (r+1)*nq/P) (one all-to-all, (P-1)/P x nq*k*8 B received per
  rank instead of (P-1) x), merges them there and returns that slice -- or
  the assembled result when ``gather=True`` (one all-gather of the final
  8*k*nq/P bytes per rank).

The local join and merge default to the CUDA library; tests may inject other
callables to exercise the orchestration on CPU with the gloo backend.
"""
from __future__ import annotations

import math

import torch
import torch.distributed as dist

from . import join as _cuda_join
from . import merge_partials as _cuda_merge
from . import merge_partials_ptrs as _cuda_merge_ptrs


def shard_bounds(n: int, world: int, rank: int):
    """Contiguous, balanced [lo, hi) of rank among world over n items."""
    base, rem = divmod(n, world)
    lo = rank * base + min(rank, rem)
    return lo, lo + base + (1 if rank < rem else 0)


def _world(group):
    if not dist.is_available() or not dist.is_initialized():
        return 1, 0  # single process: every collective below is skipped
    return dist.get_world_size(group), dist.get_rank(group)


def join_query_sharded(Q, T, k: int, *, group=None, self_join: bool | None = None, gather: bool = True,
                       local_join=None, partition: str = "clusters", **opts):
    """Query-sharded join. Returns (idx, dist) for the rank's rows (gather=False:
    full-size buffers with -1 / 0 in rows of other ranks) or the assembled
    full result on every rank (gather=True, one collective).

    partition="clusters" (default): every rank clusters all of Q (identical,
    deterministic) and takes the query clusters c % P == rank. "rows" (Q != T
    only): rank r clusters and joins the contiguous rows [r nq/P, (r+1) nq/P)
    -- no replicated query build, but measured on C4 (tools/shard_balance.py,
    one GPU per rank's share) a rank's slice can hold outlier queries whose
    near-brute-force scans run on one warp each (P = 8: 1.58 s max over ranks
    vs 46 ms with cluster interleaving)."""
    world, rank = _world(group)
    local_join = local_join or _cuda_join
    if self_join is None:
        self_join = Q is T
    nq = Q.shape[0]
    if self_join or partition == "clusters":
        idx = torch.full((nq, k), -1, dtype=torch.int32, device=Q.device)
        dst = torch.zeros((nq, k), dtype=torch.float32, device=Q.device)
        local_join(Q, Q if self_join else T, k, out=(idx, dst), shard_rank=rank, shard_count=world, **opts)
    else:
        lo, hi = shard_bounds(nq, world, rank)
        idx = torch.full((nq, k), -1, dtype=torch.int32, device=Q.device)
        dst = torch.zeros((nq, k), dtype=torch.float32, device=Q.device)
        if hi > lo:
            # cluster the slice as finely as the whole query set would be
            # (floor(3 sqrt(nq))): the default floor(3 sqrt(nq / P)) gives
            # clusters sqrt(P) x wider, and on C4 at P = 8 a 5x larger dense-tile
            # workload (measured: tools/diag_c4_slices.py)
            lopts = dict(opts)
            if world > 1 and not lopts.get("n_clusters_q"):
                lopts["n_clusters_q"] = min(int(3.0 * math.sqrt(nq)), hi - lo)
            i, d = local_join(Q[lo:hi].contiguous(), T, k, **lopts)[:2]
            idx[lo:hi] = i
            dst[lo:hi] = d
    if not gather or world == 1:
        return idx, dst
    if not self_join and partition != "clusters":
        # contiguous row slices: one all-gather of the (padded) slices
        splits = [shard_bounds(nq, world, r) for r in range(world)]
        cap = max(h - l for l, h in splits)
        lo, hi = splits[rank]
        mine = torch.zeros((cap, k, 2), dtype=torch.int32, device=Q.device)
        mine[:hi - lo, :, 0] = idx[lo:hi]
        mine[:hi - lo, :, 1] = dst[lo:hi].view(torch.int32)
        allp = torch.empty((world * cap, k, 2), dtype=torch.int32, device=Q.device)
        dist.all_gather_into_tensor(allp, mine, group=group)
        out = torch.cat([allp[r * cap:r * cap + (h - l)] for r, (l, h) in enumerate(splits)])
        return out[:, :, 0].contiguous(), out[:, :, 1].contiguous().view(torch.float32)
    # cluster-interleaved rows: each rank's rows hold (dist bits << 32 |
    # idx + 1), every other row 0, so ONE all-reduce SUM assembles both arrays
    own = idx >= 0
    packed = torch.where(own, (dst.view(torch.int32).to(torch.int64) << 32) | (idx.to(torch.int64) + 1),
                         torch.zeros((), dtype=torch.int64, device=Q.device))
    dist.all_reduce(packed, op=dist.ReduceOp.SUM, group=group)
    idx = ((packed & 0xFFFFFFFF) - 1).to(torch.int32)
    dst = (packed >> 32).to(torch.int32).view(torch.float32)
    return idx, dst


def build_index_broadcast(T, *, group=None, src: int = 0, build=None, create=None, **opts):
    """Query-sharded mode, index built ONCE: rank `src` clusters T (sknn_build)
    and every other rank receives the index arrays by torch.distributed
    broadcast (NCCL over NVLink) into an empty index of the same geometry
    (sknn_index_create) -- instead of every rank rebuilding it (SURVEY §8(e)
    "Measure both"). Returns the rank's Index; query it with self_query=1
    for a self-join. `build`/`create` may be injected (tests)."""
    from . import Index
    world, rank = _world(group)
    build = build or (lambda X, **o: Index(X, **o))
    create = create or (lambda nt, d, mt, **o: Index.create(nt, d, mt, **o))
    if rank == src:
        ix = build(T, **opts)
        inf = ix.info()
        geom = torch.tensor([inf["nt"], inf["d"], inf["mt"]], dtype=torch.int64, device=T.device)
    else:
        geom = torch.zeros(3, dtype=torch.int64, device=T.device)
    if world > 1:
        dist.broadcast(geom, src, group=group)
    if rank != src:
        ix = create(int(geom[0]), int(geom[1]), int(geom[2]), **opts)
    if world > 1:
        for buf in ix.arrays():
            dist.broadcast(buf, src, group=group)
    return ix


def join_query_sharded_index(index, Q, k: int, *, group=None, out=None, **opts):
    """Query-sharded self-join against a shared index (build_index_broadcast):
    each rank runs sknn_query over the query clusters c with c % P == rank;
    no data-path collective. Returns the full-size buffers (rows of other
    ranks untouched)."""
    world, rank = _world(group)
    return index.query(Q, k, out=out, self_query=1, shard_rank=rank, shard_count=world, **opts)


def aligned_bounds(n: int, world: int, rank: int, align: int = 8):
    """shard_bounds with every interior boundary rounded down to a multiple of
    `align` (the sharded build's row ranges)."""
    lo = (shard_bounds(n, world, rank)[0] // align) * align if rank > 0 else 0
    hi = (shard_bounds(n, world, rank)[1] // align) * align if rank < world - 1 else n
    return lo, hi


def build_index_sharded(X, *, group=None, assign_shard=None, from_assignment=None, **opts):
    """Cluster a point set every rank holds with the FINAL assignment pass
    sharded (NEXT-1, SURVEY §8(e) "sharded Q clustering"): each rank runs the
    landmark sampler and the Lloyd passes (deterministic, identical on every
    rank, on strided samples for dp <= 32) and assigns only its rows
    aligned_bounds(n, P, r) to the final centers (sknn_build_assign_shard);
    one all-reduce SUM per array assembles the assignment (other ranks' rows
    are zero) and every rank turns it into the same index
    (sknn_build_from_assignment) -- identical to sknn_build's. The
    functions may be injected (tests)."""
    from . import Index, build_assign_shard
    assign_shard = assign_shard or build_assign_shard
    from_assignment = from_assignment or (lambda X_, c, i, d, **o: Index.from_assignment(X_, c, i, d, **o))
    world, rank = _world(group)
    lo, hi = aligned_bounds(X.shape[0], world, rank)
    centers, cid, dst = assign_shard(X, lo, hi, **opts)
    if world > 1:
        dist.all_reduce(cid, op=dist.ReduceOp.SUM, group=group)
        dist.all_reduce(dst, op=dist.ReduceOp.SUM, group=group)
    return from_assignment(X, centers, cid, dst, **opts)


def target_shard_partials_global_ub(Q, T_shard, k: int, shard_offset: int, *, group=None, qindex=None, **opts):
    """Partial k-lists of ALL queries against this rank's target shard, pruned
    with the GLOBAL level-1 bound: every rank clusters Q
    identically (seeded; or pass a prebuilt `qindex`), computes the calUB of
    each query cluster against its shard (sknn_level1_bounds), the bounds are
    combined by one all-reduce MIN (mq floats: a shard's k-th distance is >=
    the global one, so every rank's bound is a global bound), and the join runs
    with the tightest one (sknn_join_indexed with ub_in). Rows may hold fewer
    than k real entries (+inf / -1 placeholders); the merged result is exact.
    Returns (idx, d2) with global indices."""
    from . import Index, join_indexed, level1_bounds
    bopts = {kk: v for kk, v in opts.items() if kk in ("lloyd_iters", "landmark_trials", "seed", "n_clusters_t")}
    shard_q = opts.pop("shard_q_build", False)
    if qindex is None and shard_q:  # every rank clusters Q, the final assignment pass split over the ranks
        qindex = build_index_sharded(Q, group=group, **bopts)
    qix = qindex or Index(Q, **bopts)
    tix = Index(T_shard)
    ub = level1_bounds(qix, tix, k)
    if dist.is_initialized() and dist.get_world_size(group) > 1:
        dist.all_reduce(ub, op=dist.ReduceOp.MIN, group=group)
    return join_indexed(qix, tix, k, out_squared=1, index_base=int(shard_offset), ub_in=ub, **opts)[:2]


def _exchange_pruned(pidx, pd2, k, splits, rank, world, group):
    """all_to_all of the partial lists with every entry above the query's
    minimum over ranks of the local k-th squared distance dropped (NEXT-1).
    Exact: the rank holding that minimum has k entries at or below it, so an
    entry strictly above it is never among the k smallest keys; entries equal
    to it are kept (ties are decided by the index in the merge). Returns the
    receiver's [world, mine, k] lists padded with (+inf, -1), the merge's input."""
    dev = pd2.device
    nq = pd2.shape[0]
    kth = pd2[:, k - 1].contiguous()  # sorted lists: the local k-th (+inf when short)
    dist.all_reduce(kth, op=dist.ReduceOp.MIN, group=group)
    keep = pd2 <= kth[:, None]
    counts = keep.sum(1, dtype=torch.int32)
    lo, hi = splits[rank]
    mine = hi - lo
    # per-query survivor counts of my rows from every rank (fixed sizes)
    rcounts = torch.empty((world, mine), dtype=torch.int32, device=dev)
    dist.all_to_all_single(rcounts.view(-1), counts, [mine] * world, [h - l for l, h in splits], group=group)
    send_tot = [int(counts[l:h].sum()) for l, h in splits]
    recv_tot = [int(x) for x in rcounts.sum(1).tolist()]
    # survivors in row-major order, so each destination's block is contiguous
    vals_d = pd2[keep].contiguous()
    vals_i = pidx[keep].contiguous()
    got_d = torch.empty(sum(recv_tot), dtype=torch.float32, device=dev)
    got_i = torch.empty(sum(recv_tot), dtype=torch.int32, device=dev)
    dist.all_to_all_single(got_d, vals_d, recv_tot, send_tot, group=group)
    dist.all_to_all_single(got_i, vals_i, recv_tot, send_tot, group=group)
    out_d = torch.full((world, mine, k), float("inf"), dtype=torch.float32, device=dev)
    out_i = torch.full((world, mine, k), -1, dtype=torch.int32, device=dev)
    if mine > 0:
        c = rcounts.view(-1).to(torch.int64)                       # [world * mine] row lengths
        row = torch.repeat_interleave(torch.arange(world * mine, device=dev), c)
        start = torch.cumsum(c, 0) - c
        col = torch.arange(row.numel(), device=dev) - start[row]
        out_d.view(world * mine, k)[row, col] = got_d
        out_i.view(world * mine, k)[row, col] = got_i
    return out_i, out_d, int(sum(send_tot))


def _exchange_peer(Q, T_shard, k, shard_offset, group, world, rank, local_join, out_squared, gather, opts):
    """exchange="peer" (NEXT-1, the fused peer-memory merge): every rank's
    partial lists are written straight into symmetric-memory buffers (torch
    symmetric memory over NVLink), one device-side barrier orders the writes,
    and rank r's merge kernel reads its rows [r nq/P, (r+1) nq/P) of all P
    buffers in place (sknn_merge_partials_ptrs) -- no exchange collective, the
    transfer overlapped with the merge arithmetic thread by thread."""
    import torch.distributed._symmetric_memory as symm_mem
    nq = Q.shape[0]
    pg = group if group is not None else dist.group.WORLD
    bi = symm_mem.empty((nq, k), dtype=torch.int32, device=Q.device)
    bd = symm_mem.empty((nq, k), dtype=torch.float32, device=Q.device)
    local_join(Q, T_shard, k, out=(bi, bd), out_squared=1, index_base=int(shard_offset), **opts)
    hi_ = symm_mem.rendezvous(bi, pg)
    hd = symm_mem.rendezvous(bd, pg)
    hd.barrier(channel=0)  # every rank's lists are written
    splits = [shard_bounds(nq, world, r) for r in range(world)]
    lo, hi = splits[rank]
    ri, rd = _cuda_merge_ptrs(hi_.buffer_ptrs, hd.buffer_ptrs, nq, lo, hi - lo, k, out_squared=out_squared,
                              device=Q.device)
    hd.barrier(channel=0)  # every rank is done reading before the buffers are released
    if not gather:
        return ri, rd
    cap = max(h - l for l, h in splits)
    pad_i = torch.full((cap, k), -1, dtype=torch.int32, device=Q.device)
    pad_d = torch.zeros((cap, k), dtype=torch.float32, device=Q.device)
    pad_i[:hi - lo] = ri
    pad_d[:hi - lo] = rd
    all_i = torch.empty((world * cap, k), dtype=torch.int32, device=Q.device)
    all_d = torch.empty((world * cap, k), dtype=torch.float32, device=Q.device)
    dist.all_gather_into_tensor(all_i, pad_i, group=group)
    dist.all_gather_into_tensor(all_d, pad_d, group=group)
    out_i = torch.cat([all_i[r * cap:r * cap + (h - l)] for r, (l, h) in enumerate(splits)])
    out_d = torch.cat([all_d[r * cap:r * cap + (h - l)] for r, (l, h) in enumerate(splits)])
    return out_i, out_d


def join_target_sharded(Q, T_shard, k: int, shard_offset: int, *, group=None, local_join=None, merge=None,
                        out_squared: bool = False, exchange: str = "all_gather", gather: bool = True,
                        global_ub: bool = False, prune: bool = False, stats: dict | None = None, **opts):
    """Target-sharded join: local partial lists of every query against this
    rank's T_shard (global indices), exchanged and merged exactly.
    exchange="all_gather": every rank merges all nq rows (returns the full
    result). exchange="all_to_all": rank r merges only its rows
    shard_bounds(nq, P, r); gather=False returns that slice, gather=True the
    full result assembled by one all-gather of the merged slices.
    prune=True (all_to_all only, NEXT-1): one all-reduce MIN of the per-query
    local k-th distances first, then only the entries at or below it travel
    (variable-size all_to_all); `stats` (a dict) receives the entry counts.
    exchange="peer" (NCCL + NVLink, k <= 32): the lists stay in symmetric
    memory and each rank's merge kernel reads the peers' buffers directly."""
    world, rank = _world(group)
    local_join = local_join or _cuda_join
    merge = merge or _cuda_merge
    nq = Q.shape[0]
    kk = min(k, T_shard.shape[0])
    if exchange == "peer" and world > 1 and not global_ub and kk == k:
        return _exchange_peer(Q, T_shard, k, shard_offset, group, world, rank, local_join, out_squared, gather, opts)
    if global_ub:  # NEXT-1: prune every shard with the global level-1 bound
        pidx, pd2 = target_shard_partials_global_ub(Q, T_shard, kk, shard_offset, group=group, **opts)
    else:
        pidx, pd2 = local_join(Q, T_shard, kk, out_squared=1, index_base=int(shard_offset), **opts)[:2]
    if kk < k:  # a shard smaller than k: pad with +inf keys (never selected over real ones)
        pad_i = torch.full((nq, k - kk), -1, dtype=torch.int32, device=Q.device)
        pad_d = torch.full((nq, k - kk), float("inf"), dtype=torch.float32, device=Q.device)
        pidx = torch.cat([pidx, pad_i], 1)
        pd2 = torch.cat([pd2, pad_d], 1)
    if world == 1:  # one shard: its partial list is the result
        return merge(pidx.view(1, nq, k), pd2.view(1, nq, k), k, out_squared=out_squared)
    if exchange == "peer":  # (world 1, global_ub or a shard smaller than k: the all-to-all path below)
        exchange = "all_to_all"
    if exchange == "all_gather":
        all_i = torch.empty((world * nq, k), dtype=torch.int32, device=Q.device)
        all_d = torch.empty((world * nq, k), dtype=torch.float32, device=Q.device)
        dist.all_gather_into_tensor(all_i, pidx.contiguous(), group=group)
        dist.all_gather_into_tensor(all_d, pd2.contiguous(), group=group)
        return merge(all_i.view(world, nq, k), all_d.view(world, nq, k), k, out_squared=out_squared)
    if exchange != "all_to_all":
        raise ValueError("exchange must be 'all_gather' or 'all_to_all'")
    # rank r receives the partial lists of its query rows from every rank: the
    # rows are contiguous per destination, so one all_to_all_single per array
    splits = [shard_bounds(nq, world, r) for r in range(world)]
    send = [(hi - lo) * k for lo, hi in splits]
    lo, hi = splits[rank]
    mine = hi - lo
    if prune:
        recv_i, recv_d, sent = _exchange_pruned(pidx, pd2, k, splits, rank, world, group)
        if stats is not None:
            stats.update(entries_sent=sent, entries_unpruned=nq * k)
    else:
        recv_i = torch.empty((world, mine, k), dtype=torch.int32, device=Q.device)
        recv_d = torch.empty((world, mine, k), dtype=torch.float32, device=Q.device)
        dist.all_to_all_single(recv_i.view(-1), pidx.contiguous().view(-1), [mine * k] * world, send, group=group)
        dist.all_to_all_single(recv_d.view(-1), pd2.contiguous().view(-1), [mine * k] * world, send, group=group)
    if mine > 0:
        ri, rd = merge(recv_i, recv_d, k, out_squared=out_squared)
    else:
        ri = torch.empty((0, k), dtype=torch.int32, device=Q.device)
        rd = torch.empty((0, k), dtype=torch.float32, device=Q.device)
    if not gather:
        return ri, rd
    # assemble the merged slices (ragged when P does not divide nq: pad to the largest)
    cap = max(h - l for l, h in splits)
    pad_i = torch.full((cap, k), -1, dtype=torch.int32, device=Q.device)
    pad_d = torch.zeros((cap, k), dtype=torch.float32, device=Q.device)
    pad_i[:mine] = ri
    pad_d[:mine] = rd
    all_i = torch.empty((world * cap, k), dtype=torch.int32, device=Q.device)
    all_d = torch.empty((world * cap, k), dtype=torch.float32, device=Q.device)
    dist.all_gather_into_tensor(all_i, pad_i, group=group)
    dist.all_gather_into_tensor(all_d, pad_d, group=group)
    out_i = torch.cat([all_i[r * cap:r * cap + (h - l)] for r, (l, h) in enumerate(splits)])
    out_d = torch.cat([all_d[r * cap:r * cap + (h - l)] for r, (l, h) in enumerate(splits)])
    return out_i, out_d
