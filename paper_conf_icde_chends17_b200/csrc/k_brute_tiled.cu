// k_brute_tiled.cu -- the dense-only path for high dimensions (SURVEY §8(f)
// NEXT-4: "high-d (d >= 1024, arcene/dor-like) dense-only path"; Table III's
// arcene d = 10,000 and dorothea d = 100,000, where the paper
// reports its filters remove only 26.9% / 91.5% of the distances, Table IV
// P:L757-761). Every query against every target -- the elastic switch's
// "regular" branch taken for the whole join -- as a register-
// tiled SIMT contraction with the top-k fused:
//
//   * a CTA owns 64 queries x one slice of the targets; per 64 x 64 tile the
//     dimensions stream through shared memory in chunks of 32 (rows read
//     coalesced, stored dimension-major), each of 256 threads accumulates a
//     4 x 4 block of squared distances in registers, dimension by dimension in
//     ascending order with one fma each -- the same sequence d2_rows uses, so
//     the keys are bit-identical to every other path's;
//   * the pairs under a query's current k-th key are appended to a per-query
//     shared buffer; one warp per 8 queries merges them into lane-distributed
//     sorted lists (warp_insert) and republishes the k-th key;
//   * target slices (enough CTAs to fill the GPU when nq is small) write
//     partial lists of squared distances with global indices, merged exactly by
//     the partial-list merge (k_merge_tpq / k_merge, sknn_merge_partials).
//
// Bound: FMA pipe (2 flops per pair-dimension: a subtract and an fma); the
// 64 x 64 x 16 chunk reads 8 KB for 131 K flops (16 flop/B, above the 11.4
// flop/B balance of 74 TF / 6.5 TB/s).
#include <cuda_runtime.h>
#include <stdint.h>

#include <algorithm>

#include "k_scan_common.cuh"

namespace sknn {

constexpr int kBtM = 64, kBtN = 64, kBtK = 16, kBtBuf = 64;  // 41 KB of static shared memory

__global__ void __launch_bounds__(256) k_brute_tiled(const float* __restrict__ Q, int64_t nq, int ldq,
                                                     const float* __restrict__ T, int64_t nt, int ldt,
                                                     const int32_t* __restrict__ torig, int d, int k,
                                                     int nslice, int64_t slice_len, float* __restrict__ part_d2,
                                                     int32_t* __restrict__ part_idx, int64_t index_base,
                                                     unsigned long long* __restrict__ evals_out) {
    __shared__ __align__(16) float s_q[kBtK][kBtM + 4];
    __shared__ __align__(16) float s_t[kBtK][kBtN + 4];
    __shared__ key_t s_buf[kBtM][kBtBuf];
    __shared__ int s_cnt[kBtM];
    __shared__ key_t s_kth[kBtM];
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const int ty = tid >> 4, tx = tid & 15;
    const int slice = blockIdx.x % nslice;
    const int64_t q0 = (int64_t)(blockIdx.x / nslice) * kBtM;
    const int64_t t_lo = (int64_t)slice * slice_len, t_hi = std::min<int64_t>(nt, t_lo + slice_len);
    // per-warp lists: warp w keeps queries 8w .. 8w+7, list r of query i in lane r of mine[i]
    key_t mine[8];
#pragma unroll
    for (int i = 0; i < 8; ++i) mine[i] = (lane < 32 - k) ? kNegKey : kInfKey;
    if (tid < kBtM) {
        s_cnt[tid] = 0;
        s_kth[tid] = kInfKey;
    }
    unsigned long long evals = 0;
    for (int64_t tb = t_lo; tb < t_hi; tb += kBtN) {
        float acc[4][4];
#pragma unroll
        for (int u = 0; u < 4; ++u)
#pragma unroll
            for (int v = 0; v < 4; ++v) acc[u][v] = 0.f;
        // 64 rows x 16 dims of each side per chunk: thread -> 4 (row, dim) elements
        // of each side, scalar loads (rows of any d and alignment), zero past d / n;
        // the next chunk is loaded into registers while this one is computed
        constexpr int kPer = kBtM * kBtK / 256;
        float pq[kPer], pt[kPer];
        auto load = [&](int c0) {
#pragma unroll
            for (int u = 0; u < kPer; ++u) {
                const int e = tid + 256 * u;
                const int r = e / kBtK, c = e % kBtK;
                const int64_t qi = q0 + r, tj = tb + r;
                const int cc = c0 + c;
                pq[u] = (qi < nq && cc < d) ? __ldg(Q + qi * ldq + cc) : 0.f;
                pt[u] = (tj < t_hi && cc < d) ? __ldg(T + tj * ldt + cc) : 0.f;
            }
        };
        load(0);
        for (int c0 = 0; c0 < d; c0 += kBtK) {
            __syncthreads();
#pragma unroll
            for (int u = 0; u < kPer; ++u) {
                const int e = tid + 256 * u;
                s_q[e % kBtK][e / kBtK] = pq[u];
                s_t[e % kBtK][e / kBtK] = pt[u];
            }
            __syncthreads();
            if (c0 + kBtK < d) load(c0 + kBtK);
#pragma unroll 8
            for (int c = 0; c < kBtK; ++c) {
                const float4 a = *reinterpret_cast<const float4*>(&s_q[c][ty * 4]);
                const float4 b = *reinterpret_cast<const float4*>(&s_t[c][tx * 4]);
                const float av[4] = {a.x, a.y, a.z, a.w}, bv[4] = {b.x, b.y, b.z, b.w};
#pragma unroll
                for (int u = 0; u < 4; ++u)
#pragma unroll
                    for (int v = 0; v < 4; ++v) {
                        const float x = av[u] - bv[v];
                        acc[u][v] = __fmaf_rn(x, x, acc[u][v]);
                    }
            }
        }
        // candidates under the (possibly stale) k-th key of their query
#pragma unroll
        for (int u = 0; u < 4; ++u) {
            const int r = ty * 4 + u;
            const key_t kth = s_kth[r];
#pragma unroll
            for (int v = 0; v < 4; ++v) {
                const int64_t tj = tb + tx * 4 + v;
                if (q0 + r < nq && tj < t_hi) {
                    ++evals;
                    const key_t key = make_key(acc[u][v], torig ? __ldg(torig + tj) : (int)tj);
                    if (key_lt(key, kth)) {
                        const int slot = atomicAdd(&s_cnt[r], 1);
                        if (slot < kBtBuf) s_buf[r][slot] = key;
                    }
                }
            }
        }
        __syncthreads();
        // merge: warp w, its 8 queries (the buffer holds at most 64 = one tile row)
#pragma unroll
        for (int i = 0; i < 8; ++i) {
            const int r = warp * 8 + i;
            const int n = min(s_cnt[r], kBtBuf);
            key_t kth = __shfl_sync(0xffffffffu, mine[i], 31);
            for (int j = 0; j < n; ++j) {
                const key_t key = s_buf[r][j];
                if (key_lt(key, kth)) {
                    mine[i] = warp_insert(mine[i], key, lane);
                    kth = __shfl_sync(0xffffffffu, mine[i], 31);
                }
            }
            __syncwarp();
            if (lane == 0) {
                s_cnt[r] = 0;
                s_kth[r] = kth;
            }
        }
    }
    // this slice's sorted list of each query: squared distances, global indices
#pragma unroll
    for (int i = 0; i < 8; ++i) {
        const int64_t q = q0 + warp * 8 + i;
        if (q < nq && lane >= 32 - k) {
            const int r = lane - (32 - k);
            const int64_t o = ((int64_t)slice * nq + q) * k + r;
            part_d2[o] = key_d2(mine[i]);
            part_idx[o] = mine[i] == kInfKey ? -1 : (int32_t)(key_idx(mine[i]) + index_base);
        }
    }
    for (int o = 16; o > 0; o >>= 1) evals += __shfl_xor_sync(0xffffffffu, evals, o);
    if (lane == 0 && evals) atomicAdd(evals_out, evals);
}

// Dense-only join. Writes out_idx / out_dist (sqrt unless out_squared) through
// the partial merge when the targets are split over several CTAs.
// T rows at stride ldt (an index's permuted, padded rows) with torig mapping a
// row to its original index, or (torig NULL) the caller's rows at stride d.
sknn_status run_brute_tiled(Ctx& cx, const float* Q, int64_t nq, int ldq, const float* T, int64_t nt, int ldt,
                            const int32_t* torig, int d, const ScanParams& p) {
    const int k = p.k;
    if (k > 32) {
        set_last_error("the dense-only (tiled brute force) path keeps k <= 32");
        return SKNN_ERR_UNSUPPORTED;
    }
    const int64_t qtiles = (nq + kBtM - 1) / kBtM;
    const int64_t ttiles = (nt + kBtN - 1) / kBtN;
    // target slices so that about 8 CTAs per SM are available; at least one 64-target tile each
    int64_t S = std::max<int64_t>(1, (8LL * cx.num_sms + qtiles - 1) / qtiles);
    S = std::min<int64_t>(S, ttiles);
    if (S * nq * k > (int64_t)1 << 31) S = std::max<int64_t>(1, ((int64_t)1 << 31) / (nq * k));
    const int64_t slice_len = ((ttiles + S - 1) / S) * kBtN;
    S = (nt + slice_len - 1) / slice_len;
    float* pd2;
    int32_t* pidx;
    SKNN_TRY(cx.alloc_scratch((void**)&pd2, sizeof(float) * (size_t)(S * nq * k)));
    SKNN_TRY(cx.alloc_scratch((void**)&pidx, sizeof(int32_t) * (size_t)(S * nq * k)));
    const int64_t grid = qtiles * S;
    if (grid >= (1LL << 31)) {
        set_last_error("dense-only path: grid too large");
        return SKNN_ERR_UNSUPPORTED;
    }
    k_brute_tiled<<<(unsigned)grid, 256, 0, cx.stream>>>(Q, nq, ldq, T, nt, ldt, torig, d, k, (int)S, slice_len, pd2, pidx,
                                                          p.index_base, &p.counters->evals_brute);
    cx.launched();
    SKNN_TRY(cx.check_launch("dense-only tiles"));
    return run_merge(cx, pidx, pd2, (int)S, nq, k, p.out_idx, p.out_dist, p.out_squared);
}

}  // namespace sknn
