// k_level1.cu -- Step 2 of the method: level-1 (cluster-pair) filtering.
//
// One CTA per query cluster qc fuses the paper's two level-1 kernels:
//   calUB  (§II-C Step 2.1; Fig. 4 calUB/getUBs P:L275-279;
//           GPU version P:L337): pool the bounds r_q + D(qc,tc) + d(c_tc,u_i)
//           over the k members u_i closest to each target center (Eq. 4,
//           Fig. 5) and take the k-th smallest.
//           B200 form (same value, no per-thread heaps): let v0(tc) =
//           D + d(c_tc, u_0) be each cluster's smallest bound and M_k the k-th
//           smallest v0. k distinct bounds are <= M_k, so the pooled k-th
//           smallest V_k <= M_k, and every bound <= V_k belongs to a cluster
//           with v0 <= M_k. Cheaper and usually tighter: a cluster with >= k
//           members holds k distinct bounds <= D + (its k-th smallest member
//           distance), so the minimum of that over clusters (one block
//           reduction) bounds V_k too; M_k is selected only when no cluster
//           has k members. Gather the bounds <= M of the clusters with
//           v0 <= M -- the footnote's early termination -- and select
//           their k-th smallest.
//   groupFilter (Alg. 1; Fig. 4 getLB/groupFilter P:L273-277;
//           GPU version P:L339): keep tc iff lb = D - r_q - r_t <= UB
//           (reading R6, plus the R7 rounding slack). Survivors are compacted
//           with warp ballots into shared memory and sorted by (D, tc)
//           ascending -- the candidate order of pointFilter (Fig. 4 line 1,
//           P:L263) -- then written to row qc of the [mq x mt] candidate table.
// The center distances D(qc, .) are computed once into shared memory and
// reused by both substeps; no global atomics except one counter per CTA.
#include <cuda_runtime.h>
#include <stdint.h>

#include "sknn_internal.cuh"
#include "sknn_launch.h"

namespace sknn {

typedef unsigned long long u64;

constexpr int kL1Threads = 256;
constexpr int kL1Vals = 1024;  // capacity of the gathered-bounds buffer (overflow: M_k is used)

__device__ __forceinline__ void cmpx64(u64* s, int i, int p) {
    u64 a = s[i], b = s[p];
    if (b < a) { s[i] = b; s[p] = a; }
}

// ascending bitonic (flip + half-cleaner form) over S (power of two) entries
__device__ void block_sort_u64(u64* s, int S) {
    for (int k = 2, lk = 1; k <= S; k <<= 1, ++lk) {
        for (int t = threadIdx.x; t < S / 2; t += blockDim.x) {
            const int blk = t >> (lk - 1), r = t & (k / 2 - 1);  // powers of two: shifts, not divisions
            cmpx64(s, (blk << lk) + r, (blk << lk) + k - 1 - r);
        }
        __syncthreads();
        for (int j = k / 4, lj = lk - 2; j > 0; j >>= 1, --lj) {
            for (int t = threadIdx.x; t < S / 2; t += blockDim.x) {
                const int i = ((t >> lj) << (lj + 1)) + (t & (j - 1));
                cmpx64(s, i, i + j);
            }
            __syncthreads();
        }
    }
}

constexpr int kSmallSel = 64;  // a radix bin this small finishes with a warp rank-select

// k-th smallest (1-based) of n <= kSmallSel floats in shared memory, by one
// warp: the value whose stable rank is k-1 (exact, no rounding involved).
__device__ __forceinline__ float warp_rank_select(const float* v, int n, int k) {
    const int lane = threadIdx.x & 31;
    float ans = 0.f;
    bool found = false;
    for (int i = lane; i < n; i += 32) {
        const float x = v[i];
        int r = 0;
        for (int j = 0; j < n; ++j) {
            const float y = v[j];
            r += (y < x || (y == x && j < i)) ? 1 : 0;
        }
        if (r == k - 1) { ans = x; found = true; }
    }
    const unsigned m = __ballot_sync(0xffffffffu, found);
    return __shfl_sync(0xffffffffu, ans, __ffs(m) - 1);
}

// k-th smallest (1-based) of n non-negative floats in shared memory: MSB-first
// radix select on the IEEE bits (monotone for x >= 0), 8 bits per round;
// once the bin that holds rank k has at most kSmallSel values they are
// compacted into `small` and warp 0 finishes with a rank-select. Returns +inf
// when n < k. All threads of the block must call it.
__device__ float block_kth_smallest(const float* vals, int n, int k, int* s_hist, int* s_sel, float* small) {
    if (n < k) return __int_as_float(0x7f800000);
    if (n <= kSmallSel) {
        float r = 0.f;
        if (threadIdx.x < 32) {
            r = warp_rank_select(vals, n, k);
            if (threadIdx.x == 0) small[kSmallSel] = r;
        }
        __syncthreads();
        r = small[kSmallSel];
        __syncthreads();
        return r;
    }
    uint32_t prefix = 0;
    int kk = k;
    for (int shift = 24; shift >= 0; shift -= 8) {
        const uint32_t mask = shift == 24 ? 0u : (0xffffffffu << (shift + 8));
        for (int i = threadIdx.x; i < 256; i += blockDim.x) s_hist[i] = 0;
        __syncthreads();
        for (int i = threadIdx.x; i < n; i += blockDim.x) {
            uint32_t u = __float_as_uint(vals[i]);
            if ((u & mask) == (prefix & mask)) atomicAdd(&s_hist[(u >> shift) & 255u], 1);
        }
        __syncthreads();
        if (threadIdx.x < 32) {  // warp 0: the bin that holds rank kk
            int c[8], tot = 0;
#pragma unroll
            for (int j = 0; j < 8; ++j) { c[j] = s_hist[threadIdx.x * 8 + j]; tot += c[j]; }
            int incl = tot;
            for (int o = 1; o < 32; o <<= 1) {
                int t = __shfl_up_sync(0xffffffffu, incl, o);
                if ((int)threadIdx.x >= o) incl += t;
            }
            const int excl = incl - tot;
            if (excl < kk && kk <= incl) {
                int run = excl, bin = threadIdx.x * 8, cnt = c[0];
#pragma unroll
                for (int j = 0; j < 8; ++j) {
                    if (run + c[j] >= kk) { bin = threadIdx.x * 8 + j; cnt = c[j]; break; }
                    run += c[j];
                }
                s_sel[0] = bin;
                s_sel[1] = kk - run;
                s_sel[2] = cnt;
                s_sel[3] = 0;
            }
        }
        __syncthreads();
        prefix |= uint32_t(s_sel[0]) << shift;
        kk = s_sel[1];
        const int cnt = s_sel[2];
        if (shift > 0 && cnt <= kSmallSel) {
            const uint32_t m2 = 0xffffffffu << shift;
            __syncthreads();
            for (int i = threadIdx.x; i < n; i += blockDim.x) {
                const float x = vals[i];
                if ((__float_as_uint(x) & m2) == prefix) small[atomicAdd(&s_sel[3], 1)] = x;
            }
            __syncthreads();
            float r = 0.f;
            if (threadIdx.x < 32) {
                r = warp_rank_select(small, cnt, kk);
                if (threadIdx.x == 0) small[kSmallSel] = r;
            }
            __syncthreads();
            r = small[kSmallSel];
            __syncthreads();
            return r;
        }
        __syncthreads();
    }
    return __uint_as_float(prefix);
}

// ascending bitonic sort of one key per lane across the warp
__device__ __forceinline__ u64 warp_sort_u64(u64 v, int lane) {
#pragma unroll
    for (int k = 2; k <= 32; k <<= 1) {
#pragma unroll
        for (int j = k >> 1; j > 0; j >>= 1) {
            const u64 o = __shfl_xor_sync(0xffffffffu, v, j);
            const bool up = (lane & k) == 0 || k == 32;
            const bool lower = (lane & j) == 0;
            v = (lower == up) ? (o < v ? o : v) : (o > v ? o : v);
        }
    }
    return v;
}

// d(c_tc, u_k): the k-th smallest member distance of every target cluster
// (+inf with fewer than k members) -- the single-cluster bound of calUB
__global__ void k_kth_member(const int4* __restrict__ tinfo, const float* __restrict__ tdist, int mt, int k,
                             float* __restrict__ tdk) {
    const int tc = blockIdx.x * blockDim.x + threadIdx.x;
    if (tc >= mt) return;
    const int4 ti = tinfo[tc];
    tdk[tc] = ti.y - ti.x >= k ? tdist[ti.y - k] : __int_as_float(0x7f800000);
}

__global__ void __launch_bounds__(kL1Threads) k_level1(
    const float* __restrict__ qcent, const float* __restrict__ qrad, const int32_t* __restrict__ qoff,
    const float* __restrict__ tcent, const int4* __restrict__ tinfo, const float* __restrict__ tdk,
    const float* __restrict__ tdist, int mt, int dp, int row_in_smem, int k, float eta, int keys_cap, int shard_rank,
    int shard_count, int dense_mode, float dense_tau, const float* __restrict__ cq_o,
    const float* __restrict__ ct_o, float dense_eps, const float* __restrict__ ub_in, float* __restrict__ ub_out,
    int32_t* __restrict__ cand,
    int32_t* __restrict__ cand_count, float* __restrict__ cand_D, int32_t* __restrict__ dcand,
    int32_t* __restrict__ dcount, unsigned long long* __restrict__ work,
    Counters* __restrict__ counters) {
    extern __shared__ __align__(16) unsigned char smem[];
    u64* s_keys = reinterpret_cast<u64*>(smem);                               // keys_cap (>= mt) entries
    float* s_D = reinterpret_cast<float*>(smem + sizeof(u64) * keys_cap);     // [mt] center distances
    const int mt4 = (mt + 3) & ~3;                                            // keep 16-byte alignment
    float* s_v = s_D + mt4;                                                   // [max(mt4, kL1Vals)] bounds
    float* s_qc = s_v + max(mt4, kL1Vals);                                    // [dp], float4-aligned
    __shared__ int s_cnt;
    __shared__ int s_hist[256];
    __shared__ int s_sel[4];
    __shared__ float s_small[kSmallSel + 1];

    const int qc = blockIdx.x;
    const int qsize = qoff[qc + 1] - qoff[qc];
    if (qsize == 0 || (shard_count > 1 && qc % shard_count != shard_rank)) {
        if (threadIdx.x == 0) {  // +inf: neutral for a minimum over ranks (target sharding)
            ub_out[qc] = __int_as_float(0x7f800000); cand_count[qc] = 0; dcount[qc] = 0; work[qc] = 0;
        }
        return;
    }
    // the query cluster's center row: staged in shared memory when it fits
    // (row_in_smem, decided by the launcher), else read through L1 (high d)
    const float* qrow = row_in_smem ? s_qc : qcent + (int64_t)qc * dp;
    if (row_in_smem)
        for (int i = threadIdx.x; i < dp; i += blockDim.x) s_qc[i] = qcent[(int64_t)qc * dp + i];
    if (threadIdx.x == 0) s_cnt = 0;
    __syncthreads();
    const float rq = qrad[qc];
    const float INF = __int_as_float(0x7f800000);

    // ---- calUB (Step 2.1) ----
    // v0(tc) = D + smallest member distance (the member closest to c_tc)
    // m1(tc) = D + k-th smallest member distance: one cluster with >= k
    // members alone holds k distinct bounds <= m1, so min m1 >= V_k as well
    __shared__ unsigned s_m1;
    if (threadIdx.x == 0) s_m1 = __float_as_uint(INF);
    __syncthreads();
    float m1 = INF;
    // independent loads only (cluster summary, k-th member distance, center
    // row), unrolled so several clusters' loads are in flight per thread
#pragma unroll 4
    for (int tc = threadIdx.x; tc < mt; tc += blockDim.x) {
        const float dmin = __int_as_float(__ldg(&tinfo[tc].w));  // +inf if empty
        const float dk = __ldg(tdk + tc);                        // +inf if fewer than k members
        const float D = __fsqrt_rn(d2_rows(qrow, tcent + (int64_t)tc * dp, dp));
        s_D[tc] = D;
        s_v[tc] = D + dmin;
        m1 = fminf(m1, D + dk);
    }
    for (int o = 16; o > 0; o >>= 1) m1 = fminf(m1, __shfl_xor_sync(0xffffffffu, m1, o));
    if ((threadIdx.x & 31) == 0) atomicMin(&s_m1, __float_as_uint(m1));  // m1 >= 0: bits order like values
    __syncthreads();
    // gather threshold: the tighter of min m1 (no selection needed) and, only
    // when no cluster has k members, the k-th smallest v0 (radix select)
    float Mk = __uint_as_float(s_m1);
    if (Mk == INF) Mk = block_kth_smallest(s_v, mt, k, s_hist, s_sel, s_small);
    // gather every bound <= M_k of the clusters with v0 <= M_k
    for (int tc = threadIdx.x; tc < mt; tc += blockDim.x) {
        if (!(s_v[tc] <= Mk)) continue;
        const int4 ti = __ldg(tinfo + tc);
        const int lo = ti.x, hi = ti.y;
        const float D = s_D[tc];
        const int cnt = min(k, hi - lo);
        // members closest to the center first; batches of 8 independent loads
        for (int i0 = 0; i0 < cnt; i0 += 8) {
            float dv[8];
#pragma unroll
            for (int u = 0; u < 8; ++u) dv[u] = (i0 + u < cnt) ? __ldg(tdist + hi - 1 - i0 - u) : __int_as_float(0x7f800000);
            // the bounds grow along the batch: keep its prefix <= M_k with ONE
            // shared-memory atomic per batch (not one per bound: ncu showed the
            // CTAs serialised on that counter)
            int nkeep = 0;
#pragma unroll
            for (int u = 0; u < 8; ++u) nkeep += (D + dv[u] <= Mk) ? 1 : 0;
            if (nkeep == 0) break;
            const int pos = atomicAdd(&s_cnt, nkeep);
#pragma unroll
            for (int u = 0; u < 8; ++u)
                if (u < nkeep && pos + u < kL1Vals) s_keys[pos + u] = u64(__float_as_uint(D + dv[u]));
            if (nkeep < 8) break;  // later bounds only grow
        }
    }
    __syncthreads();
    const int nv = s_cnt;
    // stage the gathered values as floats (alias-free copy into s_v)
    for (int i = threadIdx.x; i < min(nv, kL1Vals); i += blockDim.x) s_v[i] = __uint_as_float(uint32_t(s_keys[i]));
    __syncthreads();
    float Vk = (nv <= kL1Vals) ? block_kth_smallest(s_v, nv, k, s_hist, s_sel, s_small) : Mk;  // overflow: M_k is a valid bound
    if (!(Vk <= Mk)) Vk = Mk;
    // UB = r_q + V_k, inflated to cover the rounding of the three summed distances (R7).
    // ub_in: an external bound of the same query cluster (target-sharded mode:
    // the minimum over ranks of their local UBs -- each bounds the k-th distance
    // over ALL targets, since a shard's k-th is >= the global k-th)
    float UB = __fmul_ru(rq + Vk, 1.f + 2.f * eta);
    if (ub_in) UB = fminf(UB, __ldg(ub_in + qc));
    if (threadIdx.x == 0) {
        ub_out[qc] = UB;
        s_cnt = 0;
    }
    __syncthreads();

    // ---- groupFilter (Step 2.2, Alg. 1) ----
    for (int base = 0; base < mt; base += blockDim.x) {
        const int tc = base + threadIdx.x;
        bool keep = false;
        float D = 0.f;
        const int4 ti = tc < mt ? __ldg(tinfo + tc) : make_int4(0, 0, 0, 0);
        if (ti.x != ti.y) {
            D = s_D[tc];
            const float rt = __int_as_float(ti.z);
            const float lb = D - rq - rt;                        // getLB (Eq. 3)
            keep = ti_keep(lb, UB, D + rq + rt, eta);             // Alg. 1 line 4 (R6, R7)
        }
        const unsigned m = __ballot_sync(0xffffffffu, keep);
        int wbase = 0;
        if ((threadIdx.x & 31) == 0 && m) wbase = atomicAdd(&s_cnt, __popc(m));
        wbase = __shfl_sync(0xffffffffu, wbase, 0);
        if (keep) {
            const int pos = wbase + __popc(m & ((1u << (threadIdx.x & 31)) - 1u));
            s_keys[pos] = (u64(__float_as_uint(D)) << 32) | u64(uint32_t(tc));
        }
    }
    __syncthreads();
    const int nc = s_cnt;
    if (nc <= 32) {  // one warp sorts in registers (the common case)
        if (threadIdx.x < 32) {
            u64 v = (int)threadIdx.x < nc ? s_keys[threadIdx.x] : ~0ull;
            v = warp_sort_u64(v, threadIdx.x);
            if ((int)threadIdx.x < nc) s_keys[threadIdx.x] = v;
        }
        __syncthreads();
    } else {
        int S = 1;
        while (S < nc) S <<= 1;
        for (int i = nc + threadIdx.x; i < S; i += blockDim.x) s_keys[i] = ~0ull;
        __syncthreads();
        block_sort_u64(s_keys, S);
    }
    // elastic switch (S8): split the sorted candidates into the sparse list
    // (point-level scan, Alg. 2) and the dense-tile list (tensor cores),
    // stable in ascending D. auto: a pair is dense when a typical query's
    // member window is expected to cover at least tau of the cluster and the
    // cluster is big enough to fill tiles (cost model in DESIGN.md §6).
    int32_t* row = cand + (int64_t)qc * mt;
    int32_t* drow = dcand + (int64_t)qc * mt;
    float* Drow = cand_D + (int64_t)qc * mt;
    __shared__ int s_wcnt[2][kL1Threads / 32];
    __shared__ int s_base[2];
    __shared__ unsigned long long s_work;
    if (threadIdx.x == 0) { s_base[0] = 0; s_base[1] = 0; s_work = 0; }
    __syncthreads();
    for (int base = 0; base < nc; base += blockDim.x) {
        const int i = base + threadIdx.x;
        int tc = -1;
        bool dense = false;
        unsigned cost = 0;
        if (i < nc) {
            tc = int32_t(uint32_t(s_keys[i] & 0xffffffffu));
            // expected share of tc's members inside a typical query's Alg. 2
            // window [dq - th, dq + th] with dq ~ D and th ~ V_k (the k-th
            // nearest target bound of the cluster center, without r_q)
            const int4 ti = __ldg(tinfo + tc);
            const int sz = ti.y - ti.x;
            const float rt = __int_as_float(ti.z);
            const float Dp = s_D[tc];
            const float ov = fminf(rt, Dp + Vk) - fmaxf(0.f, Dp - Vk);
            const float share = fminf(1.f, fmaxf(0.f, ov) / fmaxf(rt, 1e-30f));
            if (dense_mode == 2) {
                dense = true;
            } else if (dense_mode == 0) {
                // and the tensor-core screen must stay selective: its error bound
                // eps (||a||^2 + ||b||^2) small against the k-th distance^2 ~ V_k^2
                const float ma = cq_o[qc] + rq, mb = ct_o[tc] + rt;
                const bool sharp = dense_eps * (ma * ma + mb * mb) <= 0.25f * Vk * Vk;
                dense = sz >= 32 && sharp && ov >= dense_tau * fmaxf(rt, 1e-30f);
            }
            // scan work estimate of a sparse pair (per query): the per-candidate
            // tests plus the expected member visits (load balancing only)
            if (!dense) cost = 4u + (unsigned)(share * (float)sz);
        }
        for (int o = 16; o > 0; o >>= 1) cost += __shfl_xor_sync(0xffffffffu, cost, o);
        if ((threadIdx.x & 31) == 0 && cost) atomicAdd(&s_work, (unsigned long long)cost);
        const unsigned md = __ballot_sync(0xffffffffu, i < nc && dense);
        const unsigned ms = __ballot_sync(0xffffffffu, i < nc && !dense);
        const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
        if (lane == 0) { s_wcnt[0][w] = __popc(ms); s_wcnt[1][w] = __popc(md); }
        __syncthreads();
        int offs = 0, offd = 0;
        for (int ww = 0; ww < w; ++ww) { offs += s_wcnt[0][ww]; offd += s_wcnt[1][ww]; }
        const unsigned below = (1u << lane) - 1u;
        if (i < nc) {
            if (dense) drow[s_base[1] + offd + __popc(md & below)] = tc;
            else {
                const int pos = s_base[0] + offs + __popc(ms & below);
                row[pos] = tc;
                Drow[pos] = __uint_as_float(uint32_t(s_keys[i] >> 32));  // center distance D (Eq. 3 per query)
            }
        }
        __syncthreads();
        if (threadIdx.x == 0) {
            int ts = 0, td = 0;
            for (int ww = 0; ww < kL1Threads / 32; ++ww) { ts += s_wcnt[0][ww]; td += s_wcnt[1][ww]; }
            s_base[0] += ts;
            s_base[1] += td;
        }
        __syncthreads();
    }
    if (threadIdx.x == 0) {
        cand_count[qc] = s_base[0];
        dcount[qc] = s_base[1];
        work[qc] = s_work;
        if (counters) {
            atomicAdd(&counters->cand_pairs, (unsigned long long)nc);
            if (s_base[1]) atomicAdd(&counters->dense_pairs, (unsigned long long)s_base[1]);
        }
    }
}

sknn_status run_level1(Ctx& cx, const Side& qs, const Side& ts, const Level1Params& p, Level1& out,
                       Counters* counters) {
    const int mq = qs.m, mt = ts.m, dp = ts.dp;
    SKNN_TRY(cx.alloc_scratch((void**)&out.ub, sizeof(float) * mq));
    SKNN_TRY(cx.alloc_scratch((void**)&out.cand, sizeof(int32_t) * (size_t)mq * mt));
    SKNN_TRY(cx.alloc_scratch((void**)&out.cand_count, sizeof(int32_t) * mq));
    SKNN_TRY(cx.alloc_scratch((void**)&out.cand_D, sizeof(float) * (size_t)mq * mt));
    SKNN_TRY(cx.alloc_scratch((void**)&out.dcand, sizeof(int32_t) * (size_t)mq * mt));
    SKNN_TRY(cx.alloc_scratch((void**)&out.dcount, sizeof(int32_t) * mq));
    SKNN_TRY(cx.alloc_scratch((void**)&out.work, sizeof(unsigned long long) * mq));
    int cap = 1;
    while (cap < mt) cap <<= 1;
    cap = std::max(cap, kL1Vals);
    const int mt4 = (mt + 3) & ~3;  // s_keys holds the gathered bounds (<= kL1Vals) before phase 2
    size_t smem = sizeof(u64) * cap + sizeof(float) * (mt4 + std::max(mt4, kL1Vals) + dp);
    const int row_in_smem = smem <= 200 * 1024 ? 1 : 0;  // high d: the center row stays in global memory
    if (!row_in_smem) smem -= sizeof(float) * dp;
    if (smem > 227 * 1024) {
        set_last_error("level-1: too many target clusters for the shared-memory candidate sort");
        return SKNN_ERR_UNSUPPORTED;
    }
    SKNN_CUDA(cudaFuncSetAttribute(k_level1, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    float* tdk;
    SKNN_TRY(cx.alloc_scratch((void**)&tdk, sizeof(float) * mt));
    k_kth_member<<<(mt + 255) / 256, 256, 0, cx.stream>>>(ts.tinfo, ts.dist, mt, p.k, tdk);
    cx.launched();
    k_level1<<<mq, kL1Threads, smem, cx.stream>>>(qs.centers, qs.radius, qs.off, ts.centers, ts.tinfo, tdk,
                                                  ts.dist, mt, dp, row_in_smem, p.k, p.eta, cap, p.shard_rank,
                                                  p.shard_count,
                                                  p.dense_mode, p.dense_tau, p.dorg ? p.dorg->cq_o : nullptr,
                                                  p.dorg ? p.dorg->ct_o : nullptr, p.dorg ? p.dorg->eps : 0.f,
                                                  p.ub_in, out.ub, out.cand, out.cand_count, out.cand_D,
                                                  out.dcand, out.dcount, out.work, counters);
    cx.launched();
    return cx.check_launch("level1");
}

}  // namespace sknn
