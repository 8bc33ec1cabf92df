#include <stdlib.h>
// k_scan.cu -- Step 3 of the method: level-2 (point-level) filtering fused
// with exact distance evaluation and per-query top-k (Alg. 2, P:L355-375;
// Fig. 4 pointFilter), plus the brute-force anchor and the partial
// list merge.
//
// Thread-data remapping (§IV-C1, Tables I-II): work is cut into
// tiles of queries of ONE query cluster, so every thread of a CTA walks the
// same candidate list in the same order. Two mappings (§IV-B2 / §IV-D3):
//   k_scan_tpq  one thread per query (query-level parallelism);
//               kNearests in registers (Fig. 8 placement).
//   k_scan_wpq  one warp per query (multi-level parallelism):
//               lanes split the member window; kNearests is lane-distributed;
//               theta is warp-uniform (the paper's shared theta via atomicMin).
// Per candidate target cluster the member window is found by binary search
// on the distance-descending member array: the skipped prefix is Alg. 2's
// `continue` region (l < -theta, line 12) and the scan stops at the first
// member with l > theta (line 10, `break`) -- re-tested as theta shrinks.
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdio.h>
#include <string.h>

#include <algorithm>
#include <vector>

#include "k_scan_common.cuh"

namespace sknn {

// -------------------------------------------------------- warp per query --
// Multi-level parallelism (§IV-B2; Fig. 8): one warp per
// query, lanes split the member window of each candidate cluster, kNearests
// is lane-distributed (lane r holds rank r) and theta is warp-uniform (the
// paper's shared theta via atomicMin becomes a shuffle). Warps fetch tiles of
// up to `tile` queries of one cluster from the atomic scheduler; no CTA
// barriers. DP > 0: the query sits in registers of every lane; DP == 0:
// runtime dp, the query is staged in shared memory per warp.
template <int DP, bool QG = false>  // QG: (runtime dp only) query rows read from global memory (high d)
__global__ void __launch_bounds__(256) k_scan_wpq(ScanArgs a) {
    extern __shared__ __align__(16) float s_q[];  // [8 warps x dp] when DP == 0
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const int ntiles = *a.ntiles;
    const int dp = DP > 0 ? DP : a.dp;
    float* sq_s = s_q + warp * (DP > 0 || QG ? 0 : dp);
    unsigned long long evals = 0, cevals = 0;
    for (;;) {
        int tile = 0;
        if (lane == 0) tile = atomicAdd(a.tile_counter, 1);
        tile = __shfl_sync(0xffffffffu, tile, 0);
        if (tile >= ntiles) break;
        const int4 tl = a.tiles[tile];
        const int qc = tl.x;
        const int qlo = a.qoff[qc], qsz = a.qoff[qc + 1] - qlo;
        const int tcount = (tl.z >> 16) & 0xff;  // single-query (outlier) tasks: 1
        const int nq_tile = min(tcount ? tcount : a.tile, qsz - tl.y);
        const float ub = a.ub[qc];
        const int ncand = a.cand_count[qc];
        const int32_t* cl = a.cand + (int64_t)qc * a.mt;
        for (int qi = 0; qi < nq_tile; ++qi) {
            const int qpos = qlo + tl.y + qi;
            float4 q[DP > 0 ? DP / 4 : 1];
            if constexpr (DP > 0) {
#pragma unroll
                for (int c = 0; c < DP / 4; ++c) q[c] = __ldg(reinterpret_cast<const float4*>(a.qrows + (int64_t)qpos * DP) + c);
            } else if constexpr (!QG) {
                __syncwarp();
                for (int c = lane; c < dp; c += 32) sq_s[c] = a.qrows[(int64_t)qpos * dp + c];
                __syncwarp();
            }
            // runtime dp: the query row staged per warp, or (high d) read through L1
            const float* sq = QG ? a.qrows + (int64_t)qpos * dp : sq_s;
            key_t mine = (lane < 32 - a.k) ? kNegKey : kInfKey;
            if (a.init_topk && a.dcount[qc] > 0 && lane >= 32 - a.k) mine = a.init_topk[(int64_t)qpos * a.k + lane - (32 - a.k)];
            key_t kth = __shfl_sync(0xffffffffu, mine, 31);
            float theta = fminf(ub, __fsqrt_ru(key_d2(kth)));
            const float rown = __ldg(a.qdist + qpos);  // d(q, c_q)
            const float* cD = a.cand_D + (int64_t)qc * a.mt;
            // the per-query 2-landmark bound (Eq. 3) of 32 candidates at once, one
            // per lane (ascending D is kept: survivors are taken lowest lane first);
            // a survivor is re-tested with the theta reached when its turn comes
            for (int c0 = 0; c0 < ncand; c0 += 32) {
                const int cme = c0 + lane;
                int tcl = 0;
                int4 til = make_int4(0, 0, 0, 0);
                float Dl = 0.f;
                bool okl = false;
                if (cme < ncand) {
                    tcl = __ldg(cl + cme);
                    til = __ldg(a.tinfo + tcl);  // {lo, hi, r_t, smallest member distance}
                    Dl = __ldg(cD + cme);
                    const float rtl = __int_as_float(til.z);
                    okl = ti_keep(Dl - rown - rtl, theta, Dl + rown + rtl, a.eta);
                }
                unsigned pend = __ballot_sync(0xffffffffu, okl);
              while (pend) {
                const int src = __ffs(pend) - 1;
                pend &= pend - 1;
                const int tc = __shfl_sync(0xffffffffu, tcl, src);
                int4 ti;
                ti.x = __shfl_sync(0xffffffffu, til.x, src);
                ti.y = __shfl_sync(0xffffffffu, til.y, src);
                ti.z = __shfl_sync(0xffffffffu, til.z, src);
                ti.w = __shfl_sync(0xffffffffu, til.w, src);
                const float D = __shfl_sync(0xffffffffu, Dl, src), rt = __int_as_float(ti.z);
                if (!ti_keep(D - rown - rt, theta, D + rown + rt, a.eta)) continue;
                const int lo = ti.x, hi = ti.y;
                float dq2;
                if constexpr (DP > 0) {
                    dq2 = d2_reg<DP>(q, a.tcent + (int64_t)tc * DP);
                } else {
                    // runtime dp: lanes split the dimensions (coalesced center row),
                    // a fixed reduction tree, lane 0's sum broadcast (warp-uniform dq;
                    // a bound input, so any fp32 order is covered by the R7 slack)
                    const float4* c4 = reinterpret_cast<const float4*>(a.tcent + (int64_t)tc * dp);
                    const float4* q4 = reinterpret_cast<const float4*>(sq);
                    float part = 0.f;
                    for (int v = lane; v < dp / 4; v += 32) part = d2_acc4(part, q4[v], __ldg(c4 + v));
                    for (int o = 16; o > 0; o >>= 1) part += __shfl_down_sync(0xffffffffu, part, o);
                    dq2 = __shfl_sync(0xffffffffu, part, 0);
                }
                const float dq = __fsqrt_rn(dq2);
                if (lane == 0) ++cevals;
                if (!ti_keep(dq - rt, theta, dq + rt, a.eta)) continue;
                const float dtmin = __int_as_float(ti.w);
                if (!ti_keep(dtmin - dq, theta, dq + dtmin, a.eta)) continue;
                const int j0 = window_start(a.tdist, lo, hi, dq, theta, a.eta);
                for (int base = j0; base < hi; base += 32) {
                    const int j = base + lane;
                    const bool valid = j < hi;
                    const float dt = valid ? __ldg(a.tdist + j) : 0.f;
                    const float l = dq - dt;
                    const bool brk = !valid || !ti_keep(l, theta, dq + dt, a.eta);
                    const unsigned bm = __ballot_sync(0xffffffffu, brk);
                    const int first = bm ? (__ffs(bm) - 1) : 32;
                    const bool ev = lane < first && ti_keep(-l, theta, dq + dt, a.eta);
                    key_t key = kInfKey;
                    if constexpr (DP > 0) {
                        if (ev) {
                            const float d2 = d2_reg<DP>(q, a.trows + (int64_t)j * DP);
                            ++evals;
                            if (d2 <= key_d2(kth)) key = make_key(d2, __ldg(a.torig + j));
                        }
                    } else if (ev) {
                        const float d2 = d2_rows(sq, a.trows + (int64_t)j * dp, dp);
                        ++evals;
                        if (d2 <= key_d2(kth)) key = make_key(d2, __ldg(a.torig + j));
                    }
                    unsigned cm = __ballot_sync(0xffffffffu, key_lt(key, kth));
                    while (cm) {
                        const int src = __ffs(cm) - 1;
                        const key_t kk = __shfl_sync(0xffffffffu, key, src);
                        mine = warp_insert(mine, kk, lane);
                        kth = __shfl_sync(0xffffffffu, mine, 31);
                        cm &= ~(1u << src);
                        cm &= __ballot_sync(0xffffffffu, key_lt(key, kth));
                    }
                    theta = fminf(ub, __fsqrt_ru(key_d2(kth)));
                    if (bm) break;
                }
              }
            }
            if (lane >= 32 - a.k) write_result(a, __ldg(a.qorig + qpos), lane - (32 - a.k), mine);
        }
    }
    add_counter(&a.counters->evals_sparse, evals);
    add_counter(&a.counters->rows_loaded, evals);
    add_counter(&a.counters->center_evals, cevals);
}

// ---------------------------------------------------------------- tiles --
// Single CTA: tiles of `tile` queries per non-empty query cluster.
__global__ void __launch_bounds__(1024) k_make_tiles(const int32_t* __restrict__ qoff, int mq, int tile,
                                                     int shard_rank, int shard_count, const int32_t* __restrict__ need,
                                                     int2* __restrict__ tiles, int* __restrict__ ntiles,
                                                     int* __restrict__ counter) {
    __shared__ int s_sum[1024];
    __shared__ int s_carry;
    if (threadIdx.x == 0) s_carry = 0;
    __syncthreads();
    for (int base = 0; base < mq; base += 1024) {
        int c = base + threadIdx.x;
        int sz = (c < mq) ? qoff[c + 1] - qoff[c] : 0;
        if (shard_count > 1 && c % shard_count != shard_rank) sz = 0;
        if (need && c < mq && need[c] == 0) sz = 0;
        int nt = (sz + tile - 1) / tile;
        s_sum[threadIdx.x] = nt;
        __syncthreads();
        for (int w = 1; w < 1024; w <<= 1) {
            int t = (threadIdx.x >= w) ? s_sum[threadIdx.x - w] : 0;
            __syncthreads();
            s_sum[threadIdx.x] += t;
            __syncthreads();
        }
        int start = s_carry + s_sum[threadIdx.x] - nt;
        for (int t = 0; t < nt; ++t) tiles[start + t] = make_int2(c, t * tile);
        __syncthreads();
        if (threadIdx.x == 1023) s_carry += s_sum[1023];
        __syncthreads();
    }
    if (threadIdx.x == 0) { *ntiles = s_carry; *counter = 0; }
}

// exclusive scan over a 1024-thread block (warp shuffles + one smem row)
__device__ __forceinline__ int block_exscan(int v, int* s_warp, int& total) {
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    int x = v;
    for (int o = 1; o < 32; o <<= 1) {
        const int y = __shfl_up_sync(0xffffffffu, x, o);
        if (lane >= o) x += y;
    }
    if (lane == 31) s_warp[w] = x;
    __syncthreads();
    if (w == 0) {
        int t = s_warp[lane];
        for (int o = 1; o < 32; o <<= 1) {
            const int y = __shfl_up_sync(0xffffffffu, t, o);
            if (lane >= o) t += y;
        }
        s_warp[lane] = t;
    }
    __syncthreads();
    const int r = (w ? s_warp[w - 1] : 0) + x - v;
    total = s_warp[31];
    __syncthreads();
    return r;
}

__device__ __forceinline__ unsigned long long block_sum_u64(unsigned long long v, unsigned long long* s_red) {
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    if (lane == 0) s_red[w] = v;
    __syncthreads();
    if (w == 0) {
        unsigned long long t = lane < (int)(blockDim.x >> 5) ? s_red[lane] : 0ull;
        for (int o = 16; o > 0; o >>= 1) t += __shfl_xor_sync(0xffffffffu, t, o);
        if (lane == 0) s_red[32] = t;
    }
    __syncthreads();
    const unsigned long long t = s_red[32];
    __syncthreads();
    return t;
}

// componentwise exclusive scan of an int4 over a 1024-thread block
__device__ __forceinline__ int4 block_exscan4(int4 v, int4* s_warp, int4& total) {
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    int4 x = v;
    for (int o = 1; o < 32; o <<= 1) {
        const int yx = __shfl_up_sync(0xffffffffu, x.x, o), yy = __shfl_up_sync(0xffffffffu, x.y, o);
        const int yz = __shfl_up_sync(0xffffffffu, x.z, o), yw = __shfl_up_sync(0xffffffffu, x.w, o);
        if (lane >= o) { x.x += yx; x.y += yy; x.z += yz; x.w += yw; }
    }
    if (lane == 31) s_warp[w] = x;
    __syncthreads();
    if (w == 0) {
        int4 t = s_warp[lane];
        for (int o = 1; o < 32; o <<= 1) {
            const int yx = __shfl_up_sync(0xffffffffu, t.x, o), yy = __shfl_up_sync(0xffffffffu, t.y, o);
            const int yz = __shfl_up_sync(0xffffffffu, t.z, o), yw = __shfl_up_sync(0xffffffffu, t.w, o);
            if (lane >= o) { t.x += yx; t.y += yy; t.z += yz; t.w += yw; }
        }
        s_warp[lane] = t;
    }
    __syncthreads();
    const int4 base = w ? s_warp[w - 1] : make_int4(0, 0, 0, 0);
    total = s_warp[31];
    return make_int4(base.x + x.x - v.x, base.y + x.y - v.y, base.z + x.z - v.z, base.w + x.w - v.w);
}

// Level-2 task list (single CTA, each thread owns <= kTaskPer consecutive
// clusters), load-balanced on the level-1 work estimate:
//  * a tile (`tile` queries of one cluster) whose estimated work exceeds both
//    total / resident warps (it alone would outlast the average warp) and 4x
//    the mean tile (measured: splitting moderate tiles costs more than the
//    balance gains) is SPLIT into S <= 32 tasks of about half the per-warp
//    average that take every S-th candidate cluster (interleaved, so each
//    task sees near and far clusters); the S tasks of a tile share the
//    queries' k-th distance bound through `theta2` and their partial lists
//    are merged by k_merge_split;
//  * order: split tasks first, then unsplit tiles heavier than W0 / 4, then
//    the rest (longest work first, so no straggler starts last).
// Split tasks are capped at `cap_split` (W0 doubles until they fit); their
// part index equals their task index. split == false (warp-per-query scan)
// keeps S = 1 and only orders.
constexpr int kTaskPer = kMaxClusters / 1024;
__global__ void __launch_bounds__(1024) k_make_tasks(const int32_t* __restrict__ qoff, int mq, int tile,
                                                     int shard_rank, int shard_count, const int32_t* __restrict__ owner,
                                                     const unsigned long long* __restrict__ work,
                                                     const int32_t* __restrict__ ccount, int slots, int cap_split,
                                                     int split, int order, int outliers, int min_split,
                                                     float wfac, float hfac,
                                                     int4* __restrict__ tasks, int* __restrict__ ntasks,
                                                     int4* __restrict__ merges, int* __restrict__ nmerges) {
    __shared__ unsigned long long s_red[33];
    __shared__ int4 s_warp4[32];
    const int per = (mq + 1023) / 1024;
    const int c0 = threadIdx.x * per;
    int nt[kTaskPer];
    unsigned long long wk[kTaskPer];
    int ncc[kTaskPer];
    unsigned long long tot = 0, ntl = 0;
#pragma unroll
    for (int u = 0; u < kTaskPer; ++u) {
        const int c = c0 + u;
        nt[u] = 0;
        wk[u] = 0;
        ncc[u] = 1;
        const bool mine = owner ? (c < mq && owner[c] == shard_rank) : !(shard_count > 1 && c % shard_count != shard_rank);
        if (u < per && c < mq && mine) {
            nt[u] = (qoff[c + 1] - qoff[c] + tile - 1) / tile;
            wk[u] = work[c];
            ncc[u] = ccount[c] > 1 ? ccount[c] : 1;
        }
        tot += (unsigned long long)nt[u] * wk[u];
        ntl += (unsigned long long)nt[u];
    }
    tot = block_sum_u64(tot, s_red);
    ntl = block_sum_u64(ntl, s_red);
    // a tile is a straggler when its work exceeds both the average per
    // resident warp and hfac x the mean tile; it is cut into pieces of
    // wfac x the average per resident warp
    const double per_slot = (double)tot / (double)slots;
    const double mean = (double)tot / (double)(ntl ? ntl : 1);
    const unsigned long long H = (unsigned long long)fmax(per_slot, hfac * mean);
    unsigned long long W0 = (unsigned long long)(per_slot * wfac);
    if (W0 < 64) W0 = 64;
    // min_split (Fig. 8): with fewer queries than r * max_cur every
    // tile is split into at least that many candidate-interleaved tasks -- the
    // paper's "several threads per query", here several warps per query tile
    auto s_of = [&](int u, unsigned long long w0) -> int {
        if (!split || nt[u] == 0) return 1;
        unsigned long long s = 1;
        if (wk[u] > H) {
            s = (wk[u] + w0 - 1) / w0;
            s = s < 32 ? (s > 2 ? s : 2) : 32;
        }
        if (s < (unsigned long long)min_split) s = (unsigned long long)min_split;
        return (int)(s < (unsigned long long)ncc[u] ? s : (unsigned long long)ncc[u]);
    };
    if (split) {
        for (int it = 0; it < 40; ++it) {
            unsigned long long n = 0;
#pragma unroll
            for (int u = 0; u < kTaskPer; ++u) {
                const int S = s_of(u, W0);
                if (S > 1) n += (unsigned long long)nt[u] * S;
            }
            n = block_sum_u64(n, s_red);
            if (n <= (unsigned long long)cap_split) break;
            W0 *= 2;
        }
    }
    // Warp-per-query scan (split == false, tile 8): the first `tile` members of
    // a cluster are its FARTHEST queries (members sort by distance descending,
    // R11) -- the outliers whose k-th neighbour is far, so their windows stay
    // wide and they approach brute force (profiled on a C4 query slice: one such
    // 8-query tile ran 878 M cycles against a 1.9 M mean, 436 ms of a 450 ms
    // scan with the GPU idle). They become single-query tasks, scheduled first.
    int nfirst[kTaskPer];
#pragma unroll
    for (int u = 0; u < kTaskPer; ++u) {
        nfirst[u] = 0;
        if (outliers && nt[u] > 0) {
            const int c = c0 + u;
            const int qsz = qoff[c + 1] - qoff[c];
            nfirst[u] = qsz < tile ? qsz : tile;
            nt[u] = (qsz - nfirst[u] + tile - 1) / tile;
        }
    }
    // bucket sizes: x = split tasks (and outlier queries), y = heavy unsplit tiles, z = the rest, w = merge entries
    int4 cnt = make_int4(0, 0, 0, 0);
#pragma unroll
    for (int u = 0; u < kTaskPer; ++u) {
        const int S = s_of(u, W0);
        cnt.x += nfirst[u];
        if (S > 1) { cnt.x += nt[u] * S; cnt.w += nt[u]; }
        else if (!order || wk[u] * 4 >= W0) cnt.y += nt[u];
        else cnt.z += nt[u];
    }
    int4 total;
    int4 off = block_exscan4(cnt, s_warp4, total);
    off.y += total.x;
    off.z += total.x + total.y;
#pragma unroll
    for (int u = 0; u < kTaskPer; ++u) {
        const int c = c0 + u;
        for (int i = 0; i < nfirst[u]; ++i) tasks[off.x + i] = make_int4(c, i, (1 << 8) | (1 << 16), -1);
        off.x += nfirst[u];
        if (nt[u] == 0) continue;
        const int S = s_of(u, W0);
        if (S > 1) {
            for (int t = 0; t < nt[u]; ++t) {
                for (int sp = 0; sp < S; ++sp) {
                    const int id = off.x + t * S + sp;
                    tasks[id] = make_int4(c, t * tile, sp | (S << 8), id);
                }
                merges[off.w + t] = make_int4(c, t * tile, S, off.x + t * S);
            }
            off.x += nt[u] * S;
            off.w += nt[u];
        } else {
            int& o = (!order || wk[u] * 4 >= W0) ? off.y : off.z;
            for (int t = 0; t < nt[u]; ++t) tasks[o + t] = make_int4(c, nfirst[u] + t * tile, 1 << 8, -1);
            o += nt[u];
        }
    }
    if (threadIdx.x == 0) {
        ntasks[0] = total.x + total.y + total.z;
        ntasks[1] = 0;
        *nmerges = total.w;
    }
}

int occupancy_grid(Ctx& cx, const void* fn, int threads, size_t smem) {
    int per_sm = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, fn, threads, smem);
    if (per_sm < 1) per_sm = 1;
    return per_sm * cx.num_sms;
}

template <int DP>
static void launch_wpq(Ctx& cx, const ScanArgs& a) {
    size_t smem = DP > 0 ? 0 : sizeof(float) * 8 * a.dp;
    if (DP == 0 && smem > 160 * 1024) {  // high d: query rows read through L1, no staging
        const int grid = occupancy_grid(cx, (const void*)k_scan_wpq<0, true>, 256, 0);
        if (a.probe_warps) {
            *a.probe_warps = grid * (256 / 32);
            return;
        }
        k_scan_wpq<0, true><<<grid, 256, 0, cx.stream>>>(a);
        return;
    }
    if (smem > 48 * 1024) cudaFuncSetAttribute(k_scan_wpq<DP>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    int grid = occupancy_grid(cx, (const void*)k_scan_wpq<DP>, 256, smem);
    if (a.probe_warps) {  // dry run: report resident warps for the task planner
        *a.probe_warps = grid * (256 / 32);
        return;
    }
    k_scan_wpq<DP><<<grid, 256, smem, cx.stream>>>(a);
}

// k > 96: warp per query with a thresholded shared-memory candidate buffer
// (k_scan_bigk.cu). Measured: k = 512 C2 133.9 -> 32.2 ms, C3 78.3 -> 15.0 ms,
// C5 2564 -> 647 ms; at k = 64 the per-thread heap (256 threads per CTA) is
// as fast on C2, 15% slower on C3 and 1.8x faster on C5, so 33 <= k <= 96 keeps
// it. SKNN_BIGK_HEAP=1 keeps the heap for every k (ablation).
bool scan_uses_bigk(int k) { return k > 96 && !getenv("SKNN_BIGK_HEAP"); }
bool scan_uses_tpq(int mapping, int dp, int k) {
    // SKNN_TPQ_HIGHD=1 (study): a forced thread mapping also for dp > 32 (the
    // runtime-dp union walk, query rows re-read from L1, member rows broadcast)
    static const bool highd = getenv("SKNN_TPQ_HIGHD") != nullptr;
    return !scan_uses_bigk(k) && ((mapping == SKNN_MAP_THREAD && (dp <= 32 || highd)) || k > 32);
}
int scan_tile_size(int mapping, int dp, int k) { return scan_uses_tpq(mapping, dp, k) ? 32 : 8; }

sknn_status run_tiles(Ctx& cx, const Side& qs, int tile, int k, int slots, int shard_rank, int shard_count,
                      Level1& l1, int fig8_width) {
    const char* ev = getenv("SKNN_SPLIT");  // ablation: SKNN_SPLIT=0 disables tile splitting
    const bool split = tile == 32 && !(ev && ev[0] == '0');  // thread-per-query scan only
    const char* eo = getenv("SKNN_TASKORDER");  // ablation: SKNN_TASKORDER=0 keeps cluster order
    const int order = (eo && eo[0] == '0') ? 0 : 1;
    const char* ew = getenv("SKNN_SPLITW");  // piece size, x total work / resident warps
    const float wfac = ew ? (float)atof(ew) : 0.5f;
    const char* eot = getenv("SKNN_OUTLIER_TASKS");  // ablation: 0 keeps 8-query first tiles (warp scan)
    const char* eh = getenv("SKNN_SPLITH");  // straggler threshold, x mean tile work
    const float hfac = eh ? (float)atof(eh) : 4.0f;
    // partial lists of split tasks: at most 2 x resident warps of them, <= 256 MB
    int cap = 0;
    if (split) {
        const int64_t per_task = (int64_t)32 * k * sizeof(key_t);
        cap = (int)std::min<int64_t>(2 * (int64_t)slots, ((int64_t)256 << 20) / per_task);
    }
    // (+ tile per cluster: the single-query outlier tasks of the warp-per-query scan)
    int64_t max_tiles = (qs.n + tile - 1) / tile + (int64_t)qs.m * (tile + 1) + cap;
    SKNN_TRY(cx.alloc_scratch((void**)&l1.tiles, sizeof(int4) * max_tiles));
    SKNN_TRY(cx.alloc_scratch((void**)&l1.ntiles, sizeof(int) * 2));
    SKNN_TRY(cx.alloc_scratch((void**)&l1.nmerges, sizeof(int)));
    if (split && cap > 0) {
        SKNN_TRY(cx.alloc_scratch((void**)&l1.merges, sizeof(int4) * cap));
        SKNN_TRY(cx.alloc_scratch((void**)&l1.part, sizeof(key_t) * (size_t)cap * 32 * k));
        SKNN_TRY(cx.alloc_scratch((void**)&l1.theta2, sizeof(unsigned) * (size_t)std::max<int64_t>(1, qs.n)));
        // 0x7f7f7f7f = 3.4e38f: "no bound yet" for the float-bits atomicMin
        SKNN_CUDA(cudaMemsetAsync(l1.theta2, 0x7f, sizeof(unsigned) * (size_t)qs.n, cx.stream));
    }
    l1.tile = tile;
    // Fig. 8 width, only while every tile's split fits the partial-list buffer
    int min_split = (split && cap > 0) ? std::min(fig8_width, 32) : 1;
    const char* ef = getenv("SKNN_FIG8");  // ablation: SKNN_FIG8=0 ignores the Fig. 8 width
    if (ef && ef[0] == '0') min_split = 1;
    while (min_split > 1 && ((qs.n + tile - 1) / tile + qs.m) * (int64_t)min_split > cap) min_split >>= 1;
    k_make_tasks<<<1, 1024, 0, cx.stream>>>(qs.off, qs.m, tile, shard_rank, shard_count, l1.owner, l1.work,
                                             l1.cand_count,
                                             slots, cap, split && cap > 0 ? 1 : 0, order,
                                             (tile == 8 && order && !scan_uses_bigk(k) && !(eot && eot[0] == '0')) ? 1 : 0,
                                             min_split,
                                             wfac, hfac, l1.tiles,
                                             l1.ntiles, l1.merges,
                                             l1.nmerges);
    cx.launched();
    if (getenv("SKNN_PLANDBG")) {  // diagnostics: the plan on stderr (synchronises)
        cudaStreamSynchronize(cx.stream);
        std::vector<unsigned long long> w(qs.m);
        std::vector<int32_t> off(qs.m + 1), cc(qs.m);
        int nt[2] = {0, 0}, nm = 0;
        cudaMemcpy(w.data(), l1.work, sizeof(unsigned long long) * qs.m, cudaMemcpyDeviceToHost);
        cudaMemcpy(off.data(), qs.off, sizeof(int32_t) * (qs.m + 1), cudaMemcpyDeviceToHost);
        cudaMemcpy(cc.data(), l1.cand_count, sizeof(int32_t) * qs.m, cudaMemcpyDeviceToHost);
        cudaMemcpy(nt, l1.ntiles, sizeof(int) * 2, cudaMemcpyDeviceToHost);
        if (l1.nmerges) cudaMemcpy(&nm, l1.nmerges, sizeof(int), cudaMemcpyDeviceToHost);
        double tot = 0, mx = 0;
        long tiles = 0;
        for (int c = 0; c < qs.m; ++c) {
            const int t = (off[c + 1] - off[c] + tile - 1) / tile;
            tiles += t;
            tot += (double)t * (double)w[c];
            mx = std::max(mx, (double)w[c]);
        }
        fprintf(stderr, "[plan] slots=%d tiles=%ld tasks=%d split_tiles=%d tot=%.3g mean/tile=%.3g max/tile=%.3g "
                "tot/slots=%.3g\n", slots, tiles, nt[0], nm, tot, tot / std::max(1L, tiles), mx, tot / slots);
    }
    return cx.check_launch("tasks");
}

// Balanced query sharding ("whole query clusters balanced by
// estimated work"; sknn_options.shard_policy = 1). One CTA: cluster c's
// weight is |qc| x work[c] (level-1's per-query scan estimate, an integer sum,
// so every rank computes the same bits); clusters are sorted heaviest first
// (ties by id) with a shared-memory bitonic sort and dealt to ranks in snake
// order 0..P-1, P-1..0, ... (each round gives every rank one cluster, the
// heavy end alternating). Other ranks' clusters lose their dense pairs here
// (dcount = 0) so the dense-tile list skips them.
__global__ void __launch_bounds__(1024) k_shard_owner(const int32_t* __restrict__ qoff,
                                                      const unsigned long long* __restrict__ work,
                                                      int32_t* __restrict__ dcount, int mq, int P, int rank,
                                                      int32_t* __restrict__ owner) {
    extern __shared__ unsigned long long s_key[];
    int n2 = 1;
    while (n2 < mq) n2 <<= 1;
    constexpr unsigned long long kMaxW = (1ull << 50) - 1;
    for (int i = threadIdx.x; i < n2; i += blockDim.x) {
        unsigned long long key = ~0ull;
        if (i < mq) {
            unsigned long long w = (unsigned long long)(qoff[i + 1] - qoff[i]) * work[i];
            if (w > kMaxW) w = kMaxW;
            key = ((kMaxW - w) << 14) | (unsigned long long)i;  // ascending key = heaviest first, then id
        }
        s_key[i] = key;
    }
    __syncthreads();
    for (int size = 2; size <= n2; size <<= 1)
        for (int stride = size >> 1; stride > 0; stride >>= 1) {
            for (int i = threadIdx.x; i < n2; i += blockDim.x) {
                const int j = i ^ stride;
                if (j > i) {
                    const bool up = (i & size) == 0;
                    const unsigned long long a = s_key[i], b = s_key[j];
                    if ((a > b) == up) { s_key[i] = b; s_key[j] = a; }
                }
            }
            __syncthreads();
        }
    for (int i = threadIdx.x; i < mq; i += blockDim.x) {
        const int c = (int)(s_key[i] & 0x3fffull);
        const int round = i / P, j = i - round * P;
        const int r = (round & 1) ? P - 1 - j : j;
        owner[c] = r;
        if (r != rank && dcount) dcount[c] = 0;
    }
}

sknn_status run_shard_owner(Ctx& cx, const Side& qs, Level1& l1, int shard_rank, int shard_count) {
    SKNN_TRY(cx.alloc_scratch((void**)&l1.owner, sizeof(int32_t) * (size_t)std::max(1, qs.m)));
    int n2 = 1;
    while (n2 < qs.m) n2 <<= 1;
    const size_t smem = sizeof(unsigned long long) * (size_t)n2;
    if (smem > 48 * 1024) cudaFuncSetAttribute(k_shard_owner, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    k_shard_owner<<<1, 1024, smem, cx.stream>>>(qs.off, l1.work, l1.dcount, qs.m, shard_count, shard_rank, l1.owner);
    cx.launched();
    return cx.check_launch("shard owner");
}

// dense-tile work list: tiles of 128 queries of the clusters with dense pairs
sknn_status run_dense_tiles(Ctx& cx, const Side& qs, Level1& l1) {
    const int tile = 128;
    int64_t max_tiles = (qs.n + tile - 1) / tile + qs.m;
    SKNN_TRY(cx.alloc_scratch((void**)&l1.dtiles, sizeof(int2) * max_tiles));
    SKNN_TRY(cx.alloc_scratch((void**)&l1.dntiles, sizeof(int) * 2));
    k_make_tiles<<<1, 1024, 0, cx.stream>>>(qs.off, qs.m, tile, 0, 1, l1.dcount, l1.dtiles, l1.dntiles,
                                             l1.dntiles + 1);
    cx.launched();
    return cx.check_launch("dense tiles list");
}

__global__ void k_merge_split(ScanArgs a, const int4* __restrict__ merges, const int* __restrict__ nmerges);

static void dispatch_scan(Ctx& cx, const ScanArgs& a, bool tpq, int dp) {
    if (scan_uses_bigk(a.k)) {
        launch_scan_bigk(cx, a, dp);
        return;
    }
    if (tpq) {
        switch (dp) {
            case 4: launch_tpq_dp<4>(cx, a); break;
            case 8: launch_tpq_dp<8>(cx, a); break;
            case 12: launch_tpq_dp<12>(cx, a); break;
            case 16: launch_tpq_dp<16>(cx, a); break;
            case 20: launch_tpq_dp<20>(cx, a); break;
            case 24: launch_tpq_dp<24>(cx, a); break;
            case 28: launch_tpq_dp<28>(cx, a); break;
            case 32: launch_tpq_dp<32>(cx, a); break;
            default: launch_tpq_dp<0>(cx, a); break;  // dp > 32 with k > 32
        }
    } else {
        switch (dp) {
            case 4: launch_wpq<4>(cx, a); break;
            case 8: launch_wpq<8>(cx, a); break;
            case 12: launch_wpq<12>(cx, a); break;
            case 16: launch_wpq<16>(cx, a); break;
            case 20: launch_wpq<20>(cx, a); break;
            case 24: launch_wpq<24>(cx, a); break;
            case 28: launch_wpq<28>(cx, a); break;
            case 32: launch_wpq<32>(cx, a); break;
            default: launch_wpq<0>(cx, a); break;
        }
    }
}

// resident warps of the scan kernel the dispatch would launch (task planner)
int scan_resident_warps(Ctx& cx, int mapping, int dp, int k) {
    ScanArgs a{};
    a.dp = dp;
    a.k = k;
    int w = 0;
    a.probe_warps = &w;
    dispatch_scan(cx, a, scan_uses_tpq(mapping, dp, k), dp);
    return w > 0 ? w : cx.num_sms * 32;
}

ScanArgs make_scan_args(const Side& qs, const Side& ts, const Level1& l1, const ScanParams& p) {
    const int dp = ts.dp;
    ScanArgs a{};
    a.qrows = qs.rows; a.qorig = qs.orig; a.qoff = qs.off;
    a.trows = ts.rows; a.tdist = ts.dist; a.torig = ts.orig; a.toff = ts.off; a.tcent = ts.centers;
    a.ub = l1.ub; a.cand = l1.cand; a.cand_count = l1.cand_count; a.cand_D = l1.cand_D;
    a.qdist = qs.dist; a.trad = ts.radius; a.tinfo = ts.tinfo;
    a.tiles = l1.tiles; a.ntiles = l1.ntiles; a.tile_counter = l1.ntiles + 1;
    a.part = l1.part; a.theta2 = l1.theta2;
    a.init_topk = p.init_topk; a.dcount = l1.dcount;
    a.mt = ts.m; a.dp = dp; a.k = p.k; a.tile = l1.tile; a.eta = p.eta;
    a.out_squared = p.out_squared; a.index_base = p.index_base; a.out_idx = p.out_idx; a.out_dist = p.out_dist;
    a.counters = p.counters;
    return a;
}

sknn_status run_scan(Ctx& cx, const Side& qs, const Side& ts, const Level1& l1, const ScanParams& p) {
    const int dp = ts.dp;
    const bool tpq = scan_uses_tpq(p.mapping, dp, p.k);
    ScanArgs a = make_scan_args(qs, ts, l1, p);
    dispatch_scan(cx, a, tpq, dp);
    cx.launched();
    SKNN_TRY(cx.check_launch("level2 scan"));
    if (tpq && l1.merges) {
        k_merge_split<<<cx.num_sms * 4, 256, 0, cx.stream>>>(a, l1.merges, l1.nmerges);
        cx.launched();
        SKNN_TRY(cx.check_launch("merge split tasks"));
    }
    return SKNN_OK;
}

// ------------------------------------------------- basic KNN-TI (ablation) --
// The version Sweet KNN improves on (Fig. 4 pointFilter / Alg. 2, P:L273-281,
// P:L355-375; Table IV's "KNN-TI" column): one thread per query
// in INPUT order, so neighbouring threads of a warp belong to different query
// clusters and walk different candidate lists (no thread-data remapping,
// §IV-C1); each candidate cluster's members are visited from the top of the
// distance-descending array with Alg. 2's `continue` (l < -theta) and
// `break` (l > theta); kNearests is a sorted array in thread-local memory
// with an insertion shift. Level-1 (calUB + groupFilter, the candidate lists
// in ascending D) is shared with the Sweet path. Same exact keys, so the same
// result (reading R2 ties, R6 non-strict tests, R7 slack).
__global__ void k_invert_perm(const int32_t* __restrict__ orig, int64_t n, int32_t* __restrict__ pos) {
    for (int64_t p = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; p < n; p += (int64_t)gridDim.x * blockDim.x)
        pos[orig[p]] = (int32_t)p;
}

__global__ void __launch_bounds__(256) k_scan_basic(ScanArgs a, int64_t nq, int mq, const int32_t* __restrict__ pos) {
    unsigned long long evals = 0, cevals = 0, inserts = 0;
    const int dp = a.dp, k = a.k;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < nq; i += (int64_t)gridDim.x * blockDim.x) {
        const int p = __ldg(pos + i);
        int lo = 0, hi = mq;  // query cluster: the last c with qoff[c] <= p
        while (hi - lo > 1) {
            const int mid = (lo + hi) >> 1;
            if (__ldg(a.qoff + mid) <= p) lo = mid;
            else hi = mid;
        }
        const int qc = lo;
        key_t list[32];  // kNearests, ascending; list[k-1] is the k-th key (R8: (+inf, -1) start)
        for (int r = 0; r < k; ++r) list[r] = kInfKey;
        const float ub = __ldg(a.ub + qc);
        float theta = ub;
        const float* q = a.qrows + (int64_t)p * dp;
        const int ncand = __ldg(a.cand_count + qc);
        for (int c = 0; c < ncand; ++c) {
            const int tc = __ldg(a.cand + (int64_t)qc * a.mt + c);
            const float dq = __fsqrt_rn(d2_rows(q, a.tcent + (int64_t)tc * dp, dp));
            ++cevals;
            const int jlo = __ldg(a.toff + tc), jhi = __ldg(a.toff + tc + 1);
            for (int j = jlo; j < jhi; ++j) {
                const float dt = __ldg(a.tdist + j);
                const float l = dq - dt;
                if (!ti_keep(l, theta, dq + dt, a.eta)) break;      // Alg. 2 line 10
                if (!ti_keep(-l, theta, dq + dt, a.eta)) continue;  // Alg. 2 line 12
                const float d2 = d2_rows(q, a.trows + (int64_t)j * dp, dp);
                ++evals;
                const key_t key = make_key(d2, __ldg(a.torig + j));
                if (key < list[k - 1]) {  // Alg. 2 lines 15-17: kNearests.insert
                    int r = k - 1;
                    while (r > 0 && list[r - 1] > key) {
                        list[r] = list[r - 1];
                        --r;
                    }
                    list[r] = key;
                    ++inserts;
                    theta = fminf(ub, __fsqrt_ru(key_d2(list[k - 1])));
                }
            }
        }
        for (int r = 0; r < k; ++r) write_result(a, (int)i, r, list[r]);
    }
    add_counter(&a.counters->evals_sparse, evals);
    add_counter(&a.counters->rows_loaded, evals);
    add_counter(&a.counters->center_evals, cevals);
    add_counter(&a.counters->topk_inserts, inserts);
}

sknn_status run_scan_basic(Ctx& cx, const Side& qs, const Side& ts, const Level1& l1, const ScanParams& p) {
    ScanArgs a = make_scan_args(qs, ts, l1, p);
    int32_t* pos = nullptr;
    SKNN_TRY(cx.alloc_scratch((void**)&pos, sizeof(int32_t) * (size_t)qs.n));
    const int g = (int)std::min<int64_t>((qs.n + 255) / 256, (int64_t)cx.num_sms * 8);
    k_invert_perm<<<g > 0 ? g : 1, 256, 0, cx.stream>>>(qs.orig, qs.n, pos);
    cx.launched();
    SKNN_TRY(cx.check_launch("invert permutation"));
    const int grid = occupancy_grid(cx, (const void*)k_scan_basic, 256, 0);
    k_scan_basic<<<grid, 256, 0, cx.stream>>>(a, qs.n, qs.m, pos);
    cx.launched();
    return cx.check_launch("level2 scan (basic KNN-TI)");
}

// ------------------------------------------------------------ brute force --
// Every query against every target (no filtering): the correctness anchor and
// the "no pruning" reference. Warp per query, lanes stride the targets, the
// same fp32 distance and the same warp top-k as the TI path.
__global__ void __launch_bounds__(256) k_brute(const float* __restrict__ Q, int64_t nq, const float* __restrict__ T,
                                               int64_t nt, int d, ScanArgs a) {
    extern __shared__ __align__(16) float s_qb[];
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    float* sq_s = s_qb + warp * (a.q_global ? 0 : d);
    unsigned long long evals = 0;
    for (int64_t qi = (int64_t)blockIdx.x * 8 + warp; qi < nq; qi += (int64_t)gridDim.x * 8) {
        if (!a.q_global) {
            __syncwarp();
            for (int c = lane; c < d; c += 32) sq_s[c] = Q[qi * d + c];
            __syncwarp();
        }
        const float* sq = a.q_global ? Q + qi * d : sq_s;  // high d: read through L1
        key_t mine = (lane < 32 - a.k) ? kNegKey : kInfKey;
        key_t kth = kInfKey;
        for (int64_t base = 0; base < nt; base += 32) {
            const int64_t j = base + lane;
            key_t key = kInfKey;
            if (j < nt) {
                const float* t = T + j * d;
                float s = 0.f;
                for (int c = 0; c < d; ++c) {
                    float x = sq[c] - __ldg(t + c);
                    s = __fmaf_rn(x, x, s);
                }
                key = make_key(s, (int)j);
                ++evals;
            }
            unsigned cm = __ballot_sync(0xffffffffu, key_lt(key, kth));
            while (cm) {
                const int src = __ffs(cm) - 1;
                const key_t kk = __shfl_sync(0xffffffffu, key, src);
                mine = warp_insert(mine, kk, lane);
                kth = __shfl_sync(0xffffffffu, mine, 31);
                cm &= ~(1u << src);
                cm &= __ballot_sync(0xffffffffu, key_lt(key, kth));
            }
        }
        if (lane >= 32 - a.k) write_result(a, (int)qi, lane - (32 - a.k), mine);
    }
    add_counter(&a.counters->evals_brute, evals);
}

sknn_status run_brute(Ctx& cx, const float* Q, int64_t nq, const float* T, int64_t nt, int d, const ScanParams& p) {
    ScanArgs a{};
    a.k = p.k; a.out_squared = p.out_squared; a.index_base = p.index_base;
    a.out_idx = p.out_idx; a.out_dist = p.out_dist; a.counters = p.counters;
    size_t smem = sizeof(float) * 8 * d;
    a.q_global = smem > 160 * 1024 ? 1 : 0;
    if (a.q_global) smem = 0;
    if (smem > 48 * 1024) SKNN_CUDA(cudaFuncSetAttribute(k_brute, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    int64_t blocks = (nq + 7) / 8;
    int grid = (int)std::min<int64_t>(blocks, (int64_t)cx.num_sms * 8);
    k_brute<<<grid, 256, smem, cx.stream>>>(Q, nq, T, nt, d, a);
    cx.launched();
    return cx.check_launch("brute");
}

// ------------------------------------------------------ merge split tasks --
// One thread per query of a split tile: S-way merge of the tasks' sorted
// partial lists (disjoint member sets, so the keys are distinct) into the
// final k (the paper's final merge of partial heaps).
__global__ void __launch_bounds__(256) k_merge_split(ScanArgs a, const int4* __restrict__ merges,
                                                     const int* __restrict__ nmerges) {
    __shared__ unsigned short s_head[256][33];  // k <= 512
    unsigned short* head = s_head[threadIdx.x];
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const int n = *nmerges;
    for (int e = blockIdx.x * 8 + warp; e < n; e += gridDim.x * 8) {
        const int4 m = merges[e];
        const int qlo = a.qoff[m.x], qsz = a.qoff[m.x + 1] - qlo;
        const int i = m.y + lane;
        if (i >= qsz) continue;
        const int S = m.z;
        for (int s = 0; s < S; ++s) head[s] = 0;
        const int qo = __ldg(a.qorig + qlo + i);
        for (int r = 0; r < a.k; ++r) {
            key_t best = kInfKey;
            int bs = 0;
            for (int s = 0; s < S; ++s) {
                const int h = head[s];
                if (h >= a.k) continue;
                const key_t key = a.part[((int64_t)(m.w + s) * a.k + h) * 32 + lane];
                if (key < best) { best = key; bs = s; }
            }
            head[bs] += 1;
            write_result(a, qo, r, best);
        }
    }
}

// --------------------------------------------------------- merge partials --
// Warp per query, P sorted lists of k (d2, idx) keys -> the k smallest (the
// paper's final merge of per-thread sorted heaps, across ranks).
// A list is K = 32 R keys (+inf past k), key j in register j / 32 of lane
// j % 32, read coalesced. Merging the running list A with the next list B
// keeps the K smallest of their union with a bitonic step: C_j = min(A_j,
// B_{K-1-j}) holds exactly the K smallest keys as a bitonic sequence, which
// log2 K half-cleaner stages sort (distances >= 32 inside a lane's
// registers, < 32 by shuffles). (P - 1) (1 + log2 K) compare-exchanges per
// query instead of one warp insert per key.
__device__ __forceinline__ key_t shfl_key(key_t v, int src) {
    return (key_t)__shfl_sync(0xffffffffu, (unsigned long long)v, src);
}
__device__ __forceinline__ key_t shfl_xor_key(key_t v, int m) {
    return (key_t)__shfl_xor_sync(0xffffffffu, (unsigned long long)v, m);
}

template <int R>
__device__ __forceinline__ void load_list(key_t (&v)[R], const int32_t* __restrict__ pidx,
                                          const float* __restrict__ pd2, int64_t row, int k, int lane) {
#pragma unroll
    for (int r = 0; r < R; ++r) {
        const int j = r * 32 + lane;
        v[r] = j < k ? make_key(__ldg(pd2 + row + j), __ldg(pidx + row + j)) : kInfKey;
    }
}

// sort a bitonic sequence of 32 R keys ascending (key j at reg j / 32, lane j % 32)
template <int R>
__device__ __forceinline__ void bitonic_clean(key_t (&v)[R], int lane) {
#pragma unroll
    for (int h = R / 2; h >= 1; h >>= 1)  // distances 32 h: registers r and r + h of one lane
#pragma unroll
        for (int r = 0; r < R; ++r)
            if ((r & h) == 0) {
                const key_t x = v[r], y = v[r + h];
                v[r] = x < y ? x : y;
                v[r + h] = x < y ? y : x;
            }
#pragma unroll
    for (int m = 16; m >= 1; m >>= 1) {  // distances < 32: lanes l and l ^ m
        const bool upper = (lane & m) != 0;
#pragma unroll
        for (int r = 0; r < R; ++r) {
            const key_t o = shfl_xor_key(v[r], m);
            v[r] = upper ? (v[r] < o ? o : v[r]) : (v[r] < o ? v[r] : o);
        }
    }
}

template <int R>
__global__ void __launch_bounds__(256) k_merge(const int32_t* __restrict__ pidx, const float* __restrict__ pd2, int P,
                                               int64_t nq, int k, int32_t* __restrict__ out_idx,
                                               float* __restrict__ out_dist, int out_squared) {
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    for (int64_t qi = (int64_t)blockIdx.x * 8 + warp; qi < nq; qi += (int64_t)gridDim.x * 8) {
        key_t A[R], B[R];
        load_list<R>(A, pidx, pd2, qi * k, k, lane);
        if (P > 1) load_list<R>(B, pidx, pd2, (nq + qi) * k, k, lane);
        for (int p = 1; p < P; ++p) {
            key_t Bn[R];
            if (p + 1 < P) load_list<R>(Bn, pidx, pd2, ((int64_t)(p + 1) * nq + qi) * k, k, lane);  // prefetch
            // C_j = min(A_j, B_{K-1-j}); j = 32 r + l  <->  K-1-j = 32 (R-1-r) + (31-l)
#pragma unroll
            for (int r = 0; r < R; ++r) {
                const key_t b = shfl_key(B[R - 1 - r], 31 - lane);
                A[r] = b < A[r] ? b : A[r];
            }
            bitonic_clean<R>(A, lane);
            if (p + 1 < P) {
#pragma unroll
                for (int r = 0; r < R; ++r) B[r] = Bn[r];
            }
        }
#pragma unroll
        for (int r = 0; r < R; ++r) {
            const int j = r * 32 + lane;
            if (j < k) {
                const int64_t o = qi * k + j;
                const float d2 = key_d2(A[r]);
                out_dist[o] = out_squared ? d2 : __fsqrt_rn(d2);
                if (out_idx) out_idx[o] = key_idx(A[r]);
            }
        }
    }
}

// Thread per query (k <= K <= 32): the same bitonic step, but the whole list
// of K keys lives in one thread's registers, so a compare-exchange is one
// compare and four selects producing BOTH the min and the max (the warp form
// computes each side's half on its own lane, behind two shuffles). ncu of the
// warp form at C5 P = 8: ALU pipe 77%, DRAM 40% -> this form's ALU work per
// query is ~2x smaller and the kernel streams. Rows of k % 4 == 0 keys are
// read as float4 / int4 (a thread reads whole 128 B lines; the warp's other
// lanes read their own lines, so the L1 serves the 8 vector loads per line).
// One compare for both selects. Merge keys are >= 0 and their top 11 bits
// (the float d2's bits 30..20) are never all ones for a finite or +inf d2, so
// read as IEEE doubles they are finite, non-negative and order exactly like
// the integers: one DSETP (fp64 pipe) replaces the 64-bit integer compare
// pair, which the compiler also duplicates into a less-than and a
// greater-than pair when both the min and the max are selected.
__device__ __forceinline__ void cex(key_t x, key_t y, key_t& lo, key_t& hi) {
    const bool lt = __longlong_as_double(x) < __longlong_as_double(y);
    lo = lt ? x : y;
    hi = lt ? y : x;
}

template <int K>
__device__ __forceinline__ void tmerge_load(key_t (&v)[K], const int32_t* __restrict__ pidx,
                                            const float* __restrict__ pd2, int64_t row, int k, bool vec) {
    if (vec) {
        const float4* d4 = reinterpret_cast<const float4*>(pd2 + row);
        const int4* i4 = reinterpret_cast<const int4*>(pidx + row);
#pragma unroll
        for (int c = 0; c < K / 4; ++c) {
            if (4 * c < k) {
                const float4 d = __ldg(d4 + c);
                const int4 i = __ldg(i4 + c);
                v[4 * c + 0] = make_key(d.x, i.x);
                v[4 * c + 1] = make_key(d.y, i.y);
                v[4 * c + 2] = make_key(d.z, i.z);
                v[4 * c + 3] = make_key(d.w, i.w);
            } else {
                v[4 * c + 0] = v[4 * c + 1] = v[4 * c + 2] = v[4 * c + 3] = kInfKey;
            }
        }
    } else {
#pragma unroll
        for (int j = 0; j < K; ++j) v[j] = j < k ? make_key(__ldg(pd2 + row + j), __ldg(pidx + row + j)) : kInfKey;
    }
}

template <int K>
__global__ void __launch_bounds__(128) k_merge_tpq(const int32_t* __restrict__ pidx, const float* __restrict__ pd2,
                                                   int P, int64_t nq, int k, int32_t* __restrict__ out_idx,
                                                   float* __restrict__ out_dist, int out_squared, int vec) {
    for (int64_t qi = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; qi < nq; qi += (int64_t)gridDim.x * blockDim.x) {
        key_t A[K], B[K];
        tmerge_load<K>(A, pidx, pd2, qi * k, k, vec);
        for (int p = 1; p < P; ++p) {
            tmerge_load<K>(B, pidx, pd2, ((int64_t)p * nq + qi) * k, k, vec);
            // C_j = min(A_j, B_{K-1-j}): the K smallest of A u B, bitonic
#pragma unroll
            for (int j = 0; j < K; ++j)
                A[j] = __longlong_as_double(B[K - 1 - j]) < __longlong_as_double(A[j]) ? B[K - 1 - j] : A[j];
#pragma unroll
            for (int h = K / 2; h >= 1; h >>= 1)
#pragma unroll
                for (int j = 0; j < K; ++j)
                    if ((j & h) == 0) {
                        key_t lo, hi;
                        cex(A[j], A[j + h], lo, hi);
                        A[j] = lo;
                        A[j + h] = hi;
                    }
        }
        if (vec) {
            float4* od = reinterpret_cast<float4*>(out_dist + qi * k);
            int4* oi = reinterpret_cast<int4*>(out_idx ? out_idx + qi * k : nullptr);
#pragma unroll
            for (int c = 0; c < K / 4; ++c)
                if (4 * c < k) {
                    float4 d;
                    d.x = key_d2(A[4 * c + 0]);
                    d.y = key_d2(A[4 * c + 1]);
                    d.z = key_d2(A[4 * c + 2]);
                    d.w = key_d2(A[4 * c + 3]);
                    if (!out_squared) {
                        d.x = __fsqrt_rn(d.x);
                        d.y = __fsqrt_rn(d.y);
                        d.z = __fsqrt_rn(d.z);
                        d.w = __fsqrt_rn(d.w);
                    }
                    od[c] = d;
                    if (oi)
                        oi[c] = make_int4(key_idx(A[4 * c + 0]), key_idx(A[4 * c + 1]), key_idx(A[4 * c + 2]),
                                          key_idx(A[4 * c + 3]));
                }
        } else {
#pragma unroll
            for (int j = 0; j < K; ++j)
                if (j < k) {
                    const float d2 = key_d2(A[j]);
                    out_dist[qi * k + j] = out_squared ? d2 : __fsqrt_rn(d2);
                    if (out_idx) out_idx[qi * k + j] = key_idx(A[j]);
                }
        }
    }
}

// Staged form (k % 4 == 0, 16-byte aligned rows): a CTA owns 128 queries;
// list p of those queries is one contiguous [128 x k] block of d2 and of idx,
// copied with coalesced 16-byte cp.async into shared memory (3 buffers, two
// lists in flight while one is merged) at a row stride of S 16-byte units, S
// odd, so the eight threads of a 128-bit shared load phase hit eight
// different bank quads. ncu of the direct-load form at C5 P = 8: L1/TEX 99%
// busy (every warp load touches 32 lines), DRAM 55%. The result rows go out
// the same way (staged, then coalesced stores).
__device__ __forceinline__ uint32_t smem_addr_u32(const void* p) {
    return (uint32_t)__cvta_generic_to_shared(p);
}

template <int K>
struct MergeStage {
    static constexpr int kS = (K / 4) % 2 ? K / 4 : K / 4 + 1;  // row stride in 16-byte units (odd)
    static constexpr int kRowBytes = kS * 16;
    static constexpr int kArrBytes = 128 * kRowBytes;  // one array (d2 or idx) of 128 rows
    static constexpr int kBufBytes = 2 * kArrBytes;
    static constexpr int kSmem = 3 * kBufBytes;
};

// copy rows [q0, q0 + nrows) of list p (k keys per row) into buffer `buf`
template <int K>
__device__ __forceinline__ void merge_stage_load(char* buf, const int32_t* __restrict__ pidx,
                                                 const float* __restrict__ pd2, int64_t row0, int nrows, int k) {
    const int c4 = k / 4;  // 16-byte chunks per row
    const int total = nrows * c4;
    const char* gd = reinterpret_cast<const char*>(pd2 + row0 * k);
    const char* gi = reinterpret_cast<const char*>(pidx + row0 * k);
    for (int c = threadIdx.x; c < total; c += blockDim.x) {
        const int r = c / c4, col = c - r * c4;
        const uint32_t sd = smem_addr_u32(buf + r * MergeStage<K>::kRowBytes + col * 16);
        asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(sd), "l"(gd + (int64_t)c * 16));
        asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(sd + MergeStage<K>::kArrBytes),
                     "l"(gi + (int64_t)c * 16));
    }
    asm volatile("cp.async.commit_group;" ::: "memory");
}

template <int K>
__global__ void __launch_bounds__(128) k_merge_tpq_staged(const int32_t* __restrict__ pidx,
                                                          const float* __restrict__ pd2, int P, int64_t nq, int k,
                                                          int32_t* __restrict__ out_idx, float* __restrict__ out_dist,
                                                          int out_squared) {
    extern __shared__ __align__(16) char s_merge[];
    using MS = MergeStage<K>;
    const int64_t q0 = (int64_t)blockIdx.x * 128;
    const int nrows = nq - q0 < 128 ? (int)(nq - q0) : 128;
    const int t = threadIdx.x;
    const bool mine = t < nrows;
    const int c4 = k / 4;
    // prologue: lists 0, 1 (and 2) in flight; one commit group per list
#pragma unroll 1
    for (int p = 0; p < 3 && p < P; ++p)
        merge_stage_load<K>(s_merge + p * MS::kBufBytes, pidx, pd2, (int64_t)p * nq + q0, nrows, k);
    key_t A[K];
#pragma unroll 1
    for (int p = 0; p < P; ++p) {
        // groups committed so far: min(P, p + 3); list p is complete when at most
        // min(P, p + 3) - p - 1 younger groups are still pending
        const int younger = min(P, p + 3) - p - 1;
        if (younger >= 2) asm volatile("cp.async.wait_group 2;" ::: "memory");
        else if (younger == 1) asm volatile("cp.async.wait_group 1;" ::: "memory");
        else asm volatile("cp.async.wait_group 0;" ::: "memory");
        __syncthreads();
        char* buf = s_merge + (p % 3) * MS::kBufBytes;
        key_t B[K];
        if (mine) {
            const float4* d4 = reinterpret_cast<const float4*>(buf + t * MS::kRowBytes);
            const int4* i4 = reinterpret_cast<const int4*>(buf + MS::kArrBytes + t * MS::kRowBytes);
#pragma unroll
            for (int c = 0; c < K / 4; ++c) {
                if (c < c4) {
                    const float4 d = d4[c];
                    const int4 i = i4[c];
                    B[4 * c + 0] = make_key(d.x, i.x);
                    B[4 * c + 1] = make_key(d.y, i.y);
                    B[4 * c + 2] = make_key(d.z, i.z);
                    B[4 * c + 3] = make_key(d.w, i.w);
                } else {
                    B[4 * c + 0] = B[4 * c + 1] = B[4 * c + 2] = B[4 * c + 3] = kInfKey;
                }
            }
        }
        __syncthreads();  // buffer p % 3 is free again
        if (p + 3 < P) merge_stage_load<K>(buf, pidx, pd2, (int64_t)(p + 3) * nq + q0, nrows, k);
        if (!mine) continue;
        if (p == 0) {
#pragma unroll
            for (int j = 0; j < K; ++j) A[j] = B[j];
            continue;
        }
#pragma unroll
        for (int j = 0; j < K; ++j)
            A[j] = __longlong_as_double(B[K - 1 - j]) < __longlong_as_double(A[j]) ? B[K - 1 - j] : A[j];
#pragma unroll
        for (int h = K / 2; h >= 1; h >>= 1)
#pragma unroll
            for (int j = 0; j < K; ++j)
                if ((j & h) == 0) {
                    key_t lo, hi;
                    cex(A[j], A[j + h], lo, hi);
                    A[j] = lo;
                    A[j + h] = hi;
                }
    }
    // results: rows staged in buffer 0 (every load has completed), then coalesced stores
    __syncthreads();
    if (mine) {
        float4* d4 = reinterpret_cast<float4*>(s_merge + t * MS::kRowBytes);
        int4* i4 = reinterpret_cast<int4*>(s_merge + MS::kArrBytes + t * MS::kRowBytes);
#pragma unroll
        for (int c = 0; c < K / 4; ++c)
            if (c < c4) {
                float4 d = make_float4(key_d2(A[4 * c + 0]), key_d2(A[4 * c + 1]), key_d2(A[4 * c + 2]),
                                       key_d2(A[4 * c + 3]));
                if (!out_squared) {
                    d.x = __fsqrt_rn(d.x);
                    d.y = __fsqrt_rn(d.y);
                    d.z = __fsqrt_rn(d.z);
                    d.w = __fsqrt_rn(d.w);
                }
                d4[c] = d;
                i4[c] = make_int4(key_idx(A[4 * c + 0]), key_idx(A[4 * c + 1]), key_idx(A[4 * c + 2]),
                                  key_idx(A[4 * c + 3]));
            }
    }
    __syncthreads();
    float4* od = reinterpret_cast<float4*>(out_dist + q0 * k);
    int4* oi = reinterpret_cast<int4*>(out_idx ? out_idx + q0 * k : nullptr);
    for (int c = t; c < nrows * c4; c += blockDim.x) {
        const int r = c / c4, col = c - r * c4;
        od[c] = *reinterpret_cast<const float4*>(s_merge + r * MS::kRowBytes + col * 16);
        if (oi) oi[c] = *reinterpret_cast<const int4*>(s_merge + MS::kArrBytes + r * MS::kRowBytes + col * 16);
    }
}

// Peer-buffer form (sknn_merge_partials_ptrs): list p of query row q at
// d2[p] + q k -- each rank's buffer, read where it lives (over NVLink for a
// peer's), by the thread that merges the query. Thread per query, k <= 32.
struct PeerLists {
    const int32_t* idx[kMaxPeerLists];
    const float* d2[kMaxPeerLists];
};

template <int K>
__global__ void __launch_bounds__(128) k_merge_tpq_ptrs(PeerLists L, int P, int64_t row_lo, int64_t nrows, int k,
                                                        int32_t* __restrict__ out_idx, float* __restrict__ out_dist,
                                                        int out_squared, int vec) {
    for (int64_t qi = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; qi < nrows; qi += (int64_t)gridDim.x * blockDim.x) {
        const int64_t row = (row_lo + qi) * k;
        key_t A[K], B[K];
        tmerge_load<K>(A, L.idx[0], L.d2[0], row, k, vec);
        for (int p = 1; p < P; ++p) {
            tmerge_load<K>(B, L.idx[p], L.d2[p], row, k, vec);
#pragma unroll
            for (int j = 0; j < K; ++j)
                A[j] = __longlong_as_double(B[K - 1 - j]) < __longlong_as_double(A[j]) ? B[K - 1 - j] : A[j];
#pragma unroll
            for (int h = K / 2; h >= 1; h >>= 1)
#pragma unroll
                for (int j = 0; j < K; ++j)
                    if ((j & h) == 0) {
                        key_t lo, hi;
                        cex(A[j], A[j + h], lo, hi);
                        A[j] = lo;
                        A[j + h] = hi;
                    }
        }
#pragma unroll
        for (int j = 0; j < K; ++j)
            if (j < k) {
                const float d2 = key_d2(A[j]);
                out_dist[qi * k + j] = out_squared ? d2 : __fsqrt_rn(d2);
                if (out_idx) out_idx[qi * k + j] = key_idx(A[j]);
            }
    }
}

sknn_status run_merge_ptrs(Ctx& cx, const int32_t* const* part_idx, const float* const* part_d2, int P,
                           int64_t row_lo, int64_t nrows, int k, int32_t* out_idx, float* out_dist, int out_squared) {
    PeerLists L{};
    bool vec = (k % 4) == 0;
    for (int p = 0; p < P; ++p) {
        L.idx[p] = part_idx[p];
        L.d2[p] = part_d2[p];
        vec = vec && ((uintptr_t)part_idx[p] % 16) == 0 && ((uintptr_t)part_d2[p] % 16) == 0;
    }
    const int64_t blocks = (nrows + 127) / 128;
    const int grid = (int)std::max<int64_t>(1, std::min<int64_t>(blocks, (int64_t)cx.num_sms * 8));
#define SKNN_PMERGE(K) \
    k_merge_tpq_ptrs<K><<<grid, 128, 0, cx.stream>>>(L, P, row_lo, nrows, k, out_idx, out_dist, out_squared, vec ? 1 : 0)
    if (k <= 8) SKNN_PMERGE(8);
    else if (k <= 16) SKNN_PMERGE(16);
    else SKNN_PMERGE(32);
#undef SKNN_PMERGE
    cx.launched();
    return cx.check_launch("merge (peer lists)");
}

sknn_status run_merge(Ctx& cx, const int32_t* part_idx, const float* part_d2, int P, int64_t nq, int k,
                      int32_t* out_idx, float* out_dist, int out_squared) {
    const char* env = getenv("SKNN_MERGE");  // study knob for k <= 32: "warp" | "direct" | "staged"
    if (k <= 32 && !(env && !strcmp(env, "warp"))) {
        const bool vec = (k % 4) == 0 && ((uintptr_t)part_idx % 16) == 0 && ((uintptr_t)part_d2 % 16) == 0 &&
                         ((uintptr_t)out_dist % 16) == 0 && ((uintptr_t)out_idx % 16) == 0;
        const int64_t blocks = (nq + 127) / 128;
        // measured at nq = 4M, P = 8 (tools/merge_bench.py): k = 32 staged 1.84 /
        // direct 2.04 ms; k = 16 0.79 / 0.76; k = 20 1.60 / 1.05 (the staged form
        // pads rows to K = 32 and keeps 2 CTAs per SM): staged only when k == 32
        const bool staged = env ? !strcmp(env, "staged") : k == 32;
        if (vec && staged && blocks < (1ll << 31)) {
#define SKNN_SMERGE(K)                                                                                          \
    do {                                                                                                        \
        cudaFuncSetAttribute(k_merge_tpq_staged<K>, cudaFuncAttributeMaxDynamicSharedMemorySize,                 \
                             MergeStage<K>::kSmem);                                                             \
        k_merge_tpq_staged<K><<<(int)blocks, 128, MergeStage<K>::kSmem, cx.stream>>>(part_idx, part_d2, P, nq, k, \
                                                                                     out_idx, out_dist,         \
                                                                                     out_squared);              \
    } while (0)
            if (k <= 8) SKNN_SMERGE(8);
            else if (k <= 16) SKNN_SMERGE(16);
            else SKNN_SMERGE(32);
#undef SKNN_SMERGE
            cx.launched();
            return cx.check_launch("merge");
        }
        const int grid = (int)std::max<int64_t>(1, std::min<int64_t>(blocks, (int64_t)cx.num_sms * 8));
#define SKNN_TMERGE(K) \
    k_merge_tpq<K><<<grid, 128, 0, cx.stream>>>(part_idx, part_d2, P, nq, k, out_idx, out_dist, out_squared, vec)
        if (k <= 8) SKNN_TMERGE(8);
        else if (k <= 16) SKNN_TMERGE(16);
        else SKNN_TMERGE(32);
#undef SKNN_TMERGE
        cx.launched();
        return cx.check_launch("merge");
    }
    int64_t blocks = (nq + 7) / 8;
    int grid = (int)std::max<int64_t>(1, std::min<int64_t>(blocks, (int64_t)cx.num_sms * 16));
#define SKNN_MERGE(R) k_merge<R><<<grid, 256, 0, cx.stream>>>(part_idx, part_d2, P, nq, k, out_idx, out_dist, out_squared)
    if (k <= 32) SKNN_MERGE(1);
    else if (k <= 64) SKNN_MERGE(2);
    else if (k <= 128) SKNN_MERGE(4);
    else if (k <= 256) SKNN_MERGE(8);
    else SKNN_MERGE(16);
#undef SKNN_MERGE
    cx.launched();
    return cx.check_launch("merge");
}

}  // namespace sknn
