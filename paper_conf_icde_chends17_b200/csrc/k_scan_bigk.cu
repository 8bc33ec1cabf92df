// k_scan_bigk.cu -- level-2 scan for large k (33 <= k <= 512; the paper's k
// sweep up to 512, Fig. 10 / Table V), warp per query.
//
// Fig. 8 puts kNearests in shared memory while k*4 <= th1 and in
// registers or global memory beyond. On B200 a per-thread list of k = 512
// 64-bit keys (4 KB) leaves one or two warps per SM, so this path gives each
// QUERY a warp instead ("multi-level parallelism", §IV-B2) and replaces the
// per-insert kNearests update with a thresholded candidate buffer:
//   * lanes stride over the Alg. 2 window of each candidate cluster (lines
//     7-13; consecutive members: coalesced row loads) and evaluate line 15;
//   * a key below the current k-th key T (line 16) is appended to the warp's
//     shared-memory buffer (ballot + popc compaction);
//   * when the buffer holds more than CAP - 32 keys it is bitonic-sorted by
//     the warp and cut to its k smallest: T and theta = min(UB, sqrt(T))
//     (line 17, R8) tighten once per flush instead of once per insert;
//   * after the last candidate the buffer is sorted once more and its first
//     k keys are the result row.
// Exactness: every key of a target inside the final theta window passes the
// (non-increasing) threshold when it is evaluated, and each flush keeps the k
// smallest keys seen (a selection on the total order), so the row is the k
// smallest keys -- the same argument as the full filter.
#include <cuda_runtime.h>
#include <stdint.h>

#include "k_scan_common.cuh"
#include "sknn_internal.cuh"
#include "sknn_launch.h"

namespace sknn {

constexpr int kBigkWarps = 4;  // warps per CTA (buffers: 4 x CAP x 8 B of shared memory)

// ascending bitonic sort of s[0, cap) (cap a power of two) by one warp
__device__ __forceinline__ void warp_bitonic_sort(key_t* s, int cap, int lane) {
    for (int kb = 2, lk = 1; kb <= cap; kb <<= 1, ++lk) {
        for (int t = lane; t < cap / 2; t += 32) {  // flip
            const int blk = t >> (lk - 1), r = t & (kb / 2 - 1);
            const int i = (blk << lk) + r, p = (blk << lk) + kb - 1 - r;
            const key_t x = s[i], y = s[p];
            if (y < x) { s[i] = y; s[p] = x; }
        }
        __syncwarp();
        for (int j = kb / 4, lj = lk - 2; j > 0; j >>= 1, --lj) {  // half-cleaners
            for (int t = lane; t < cap / 2; t += 32) {
                const int i = ((t >> lj) << (lj + 1)) + (t & (j - 1));
                const key_t x = s[i], y = s[i + j];
                if (y < x) { s[i] = y; s[i + j] = x; }
            }
            __syncwarp();
        }
    }
}

template <int DP>
__global__ void __launch_bounds__(32 * kBigkWarps) k_scan_bigk(ScanArgs a, int cap) {
    constexpr unsigned FULL = 0xffffffffu;
    extern __shared__ __align__(16) key_t s_buf[];  // [kBigkWarps][cap]
    const int lane = threadIdx.x & 31;
    key_t* buf = s_buf + (size_t)(threadIdx.x >> 5) * cap;
    const int ntiles = *a.ntiles;
    const int k = a.k;
    unsigned long long evals = 0, cevals = 0, ins = 0;
    for (;;) {
        int tile = 0;
        if (lane == 0) tile = atomicAdd(a.tile_counter, 1);
        tile = __shfl_sync(FULL, tile, 0);
        if (tile >= ntiles) break;
        const int4 tl = a.tiles[tile];
        const int qc = tl.x;
        const int qlo = a.qoff[qc], qsz = a.qoff[qc + 1] - qlo;
        const int nq_tile = min(a.tile, qsz - tl.y);
        const int ncand = a.cand_count[qc];
        const int32_t* cl = a.cand + (int64_t)qc * a.mt;
        const float* cD = a.cand_D + (int64_t)qc * a.mt;
        const float ub = a.ub[qc];
        for (int iq = 0; iq < nq_tile; ++iq) {  // the tile's queries, one after another
            const int qpos = qlo + tl.y + iq;
            const float* qrow = a.qrows + (int64_t)qpos * a.dp;
            float4 q[DP > 0 ? DP / 4 : 1];
            if constexpr (DP > 0) {
#pragma unroll
                for (int c = 0; c < DP / 4; ++c) q[c] = __ldg(reinterpret_cast<const float4*>(qrow) + c);
            }
            auto d2q = [&](const float* t) -> float {
                if constexpr (DP > 0) return d2_reg<DP>(q, t);
                else return d2_rows(qrow, t, a.dp);
            };
            const float rown = __ldg(a.qdist + qpos);
            float theta = ub;
            float kth_d2 = __fmul_ru(ub, ub);  // gate until k keys are known (R8)
            key_t T = kInfKey;                  // the k-th key after the last flush
            int n = 0;                          // keys in the buffer (the first k sorted after a flush)
            auto flush = [&]() {
                for (int i = n + lane; i < cap; i += 32) buf[i] = kInfKey;
                __syncwarp();
                warp_bitonic_sort(buf, cap, lane);
                n = min(n, k);
                if (n == k) {
                    T = buf[k - 1];
                    if (key_d2(T) < kth_d2) {
                        kth_d2 = key_d2(T);
                        theta = fminf(ub, __fsqrt_ru(kth_d2));  // Alg. 2 line 17
                    }
                }
            };
            for (int c = 0; c < ncand; ++c) {
                const int tc = __ldg(cl + c);
                const int4 ti = __ldg(a.tinfo + tc);
                const float D = __ldg(cD + c), rt = __int_as_float(ti.z);
                if (!ti_keep(D - rown - rt, theta, D + rown + rt, a.eta)) continue;  // Eq. 3 per query
                const float dq = __fsqrt_rn(d2q(a.tcent + (int64_t)tc * a.dp));   // line 6
                ++cevals;
                const float dtmin = __int_as_float(ti.w);
                if (!ti_keep(dq - rt, theta, dq + rt, a.eta) || !ti_keep(dtmin - dq, theta, dq + dtmin, a.eta)) continue;
                const int j0 = window_start(a.tdist, ti.x, ti.y, dq, theta, a.eta);  // line 12 region ends
                const int j1 = window_end(a.tdist, j0, ti.y, dq, theta, a.eta);      // line 10 break
                for (int jb = j0; jb < j1; jb += 32) {
                    const int j = jb + lane;
                    key_t key = kInfKey;
                    if (j < j1) {
                        const float d2 = d2q(a.trows + (int64_t)j * a.dp);  // line 15
                        if (d2 <= kth_d2) {
                            key = make_key(d2, __ldg(a.torig + j));
                            if (!(key < T)) key = kInfKey;
                        }
                    }
                    evals += (j < j1);
                    const unsigned m = __ballot_sync(FULL, key != kInfKey);
                    if (m) {
                        if (key != kInfKey) buf[n + __popc(m & ((1u << lane) - 1u))] = key;
                        n += __popc(m);
                        ins += (key != kInfKey);
                        __syncwarp();
                        if (n > cap - 32) flush();
                    }
                }
            }
            flush();  // the k smallest keys, sorted
            const int qo = __ldg(a.qorig + qpos);
            for (int r = lane; r < k; r += 32) write_result(a, qo, r, buf[r]);
            __syncwarp();
        }
    }
    add_counter(&a.counters->evals_sparse, evals);
    add_counter(&a.counters->center_evals, cevals);
    add_counter(&a.counters->topk_inserts, ins);
}

int bigk_cap(int k) {
    int cap = 64;
    while (cap < 2 * k) cap <<= 1;
    return cap;
}

template <int DP>
static void launch_bigk(Ctx& cx, const ScanArgs& a) {
    const int cap = bigk_cap(a.k);
    const size_t smem = sizeof(key_t) * (size_t)cap * kBigkWarps;
    auto fn = k_scan_bigk<DP>;
    if (smem > 48 * 1024) cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    const int grid = occupancy_grid(cx, (const void*)fn, 32 * kBigkWarps, smem);
    if (a.probe_warps) {
        *a.probe_warps = grid * kBigkWarps;
        return;
    }
    fn<<<grid, 32 * kBigkWarps, smem, cx.stream>>>(a, cap);
}

void launch_scan_bigk(Ctx& cx, const ScanArgs& a, int dp) {
    switch (dp) {
        case 4: launch_bigk<4>(cx, a); break;
        case 8: launch_bigk<8>(cx, a); break;
        case 12: launch_bigk<12>(cx, a); break;
        case 16: launch_bigk<16>(cx, a); break;
        case 20: launch_bigk<20>(cx, a); break;
        case 24: launch_bigk<24>(cx, a); break;
        case 28: launch_bigk<28>(cx, a); break;
        case 32: launch_bigk<32>(cx, a); break;
        default: launch_bigk<0>(cx, a); break;
    }
}

}  // namespace sknn
