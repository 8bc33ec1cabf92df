// k_scan_tpq.cuh -- level-2 scan, one thread per query ("query level
// parallelism", Fig. 8; Alg. 2).
//
// B200 design:
//  * warp tiles: a warp owns 32 queries of ONE query cluster (thread-data
//    remapping, §IV-C1 / Tables I-II), so all lanes walk the same candidate
//    list in the same order; candidate ids are warp-uniform broadcast loads.
//  * no CTA barriers: warps fetch tiles from a device-side atomic counter
//    (dynamic scheduling), so a finished warp never waits for a slow one.
//  * kNearests in registers (Fig. 8 placement: k*4 B <= th2), sorted 64-bit
//    (d2, index) keys; the distance-only test `d2 <= kth_d2` runs first and
//    the index is loaded only for a key that can enter the list.
//  * the member loop is software-pipelined: the next member's distance (and
//    for DP <= 8 its row) is loaded before the current one is processed.
#pragma once

#include <stdlib.h>

#include "k_scan_common.cuh"

namespace sknn {

// kNearests in shared memory (Fig. 8: k*4 <= th1 = smem/SM / threads/SM,
// P:L629), laid out like the paper's Layout 2 (Fig. 6b): slot r of
// thread t at [r][t], so a warp's accesses to one slot are contiguous. Sorted
// ascending; an insertion shifts only the slots above the insertion point.
template <int STRIDE>
struct SmemTopK {
    key_t* s;
    int k;
    __device__ __forceinline__ void init(key_t* col, int k_) {
        s = col;
        k = k_;
        for (int r = 0; r < k; ++r) s[r * STRIDE] = kInfKey;
    }
    __device__ __forceinline__ key_t get(int r) const { return s[r * STRIDE]; }
    __device__ __forceinline__ void set(int r, key_t v) { s[r * STRIDE] = v; }
    // precondition: key < current k-th; returns the new k-th
    __device__ __forceinline__ key_t insert(key_t key) {
        int i = k - 1;
        while (i > 0) {
            const key_t v = s[(i - 1) * STRIDE];
            if (!(key < v)) break;
            s[i * STRIDE] = v;
            --i;
        }
        s[i * STRIDE] = key;
        return s[(k - 1) * STRIDE];
    }
};

// DP == 0: runtime dp (> 32), the query row is re-read from L1/L2 (large k only)
template <int DP, int KMAX, bool SMEM, int THREADS>
__global__ void __launch_bounds__(THREADS) k_scan_tpq(ScanArgs a) {
    extern __shared__ __align__(16) key_t s_topk[];  // [k][256] when SMEM
    const float INF = __int_as_float(0x7f800000);
    const int lane = threadIdx.x & 31;
    const int ntiles = *a.ntiles;
    unsigned long long evals = 0, cevals = 0;
    for (;;) {
        int tile = 0;
        if (lane == 0) tile = atomicAdd(a.tile_counter, 1);
        tile = __shfl_sync(0xffffffffu, tile, 0);
        if (tile >= ntiles) break;
        const int2 tl = a.tiles[tile];
        const int qc = tl.x;
        const int qlo = a.qoff[qc], qsz = a.qoff[qc + 1] - qlo;
        const int i = tl.y + lane;
        const bool active = i < qsz;
        const int qpos = qlo + (active ? i : 0);
        constexpr int QV = DP > 0 ? DP / 4 : 1;
        float4 q[QV];
        const float* qrow = a.qrows + (int64_t)qpos * a.dp;
        if constexpr (DP > 0) {
#pragma unroll
            for (int c = 0; c < DP / 4; ++c) q[c] = __ldg(reinterpret_cast<const float4*>(qrow) + c);
        }
        auto d2q = [&](const float* t) -> float {
            if constexpr (DP > 0) return d2_reg<DP>(q, t);
            else return d2_rows(qrow, t, a.dp);
        };
        RegTopK<SMEM ? 1 : KMAX> top;
        SmemTopK<THREADS> stop;
        key_t kth;
        if constexpr (SMEM) {
            stop.init(s_topk + threadIdx.x, a.k);
            kth = kInfKey;
        } else {
            top.init(a.k);
            kth = top.kth();
        }
        const float ub = a.ub[qc];
        float theta = ub;
        if (a.init_topk && a.dcount[qc] > 0) {  // continue from the dense-tile pass
            if constexpr (SMEM) {
                for (int r = 0; r < a.k; ++r) stop.set(r, a.init_topk[(int64_t)qpos * a.k + r]);
                kth = stop.get(a.k - 1);
            } else {
#pragma unroll
                for (int s = 0; s < KMAX; ++s) {
                    const int r = s - (KMAX - a.k);
                    if (r >= 0) top.a[s] = a.init_topk[(int64_t)qpos * a.k + r];
                }
                kth = top.kth();
            }
            theta = fminf(ub, __fsqrt_ru(key_d2(kth)));
        }
        float kth_d2 = key_d2(kth);
        const int ncand = a.cand_count[qc];
        const int32_t* cl = a.cand + (int64_t)qc * a.mt;
        const float* cD = a.cand_D + (int64_t)qc * a.mt;
        const float rown = __ldg(a.qdist + qpos);  // d(q, c_q)
        if (active) {
            for (int c = 0; c < ncand; ++c) {
                const int tc = __ldg(cl + c);
                // per-query 2-landmark bound (Eq. 3 with the query itself in place of
                // the query cluster's farthest member): D - d(q,c_q) - r_t <= d(q,t)
                const float D = __ldg(cD + c), rt = __ldg(a.trad + tc);
                if (!ti_keep(D - rown - rt, theta, D + rown + rt, a.eta)) continue;
                const int lo = __ldg(a.toff + tc), hi = __ldg(a.toff + tc + 1);
                const float dq = __fsqrt_rn(d2q(a.tcent + (int64_t)tc * a.dp));  // Alg. 2 line 6
                ++cevals;
                // empty window: every member distance lies in [dt_min, r_t]
                if (!ti_keep(dq - rt, theta, dq + rt, a.eta)) continue;
                const float dtmin = __ldg(a.tdist + hi - 1);
                if (!ti_keep(dtmin - dq, theta, dq + dtmin, a.eta)) continue;
                // Alg. 2 lines 7-17, visited in order of the 1-landmark lower bound
                // |l| = |dq - dt| (Eq. 1): start where dt ~ dq and walk outward on
                // both sides, always taking the side with the smaller bound, until
                // both bounds exceed theta (lines 10-13). Every member with
                // |l| <= theta is still evaluated, but near targets come first so
                // theta (line 17) tightens after a few evaluations.
                int R = window_start_geq(a.tdist, lo, hi, dq);  // first member with dt <= dq
                int L = R - 1;
                float dtL = L >= lo ? __ldg(a.tdist + L) : 0.f;
                float dtR = R < hi ? __ldg(a.tdist + R) : 0.f;
                // DP == 4: both frontier rows are kept in registers, the consumed
                // side is refilled while its distance is computed
                constexpr bool kPre = DP == 4;
                float4 rowL = make_float4(0.f, 0.f, 0.f, 0.f), rowR = rowL;
                if constexpr (kPre) {
                    if (L >= lo) rowL = __ldg(reinterpret_cast<const float4*>(a.trows) + L);
                    if (R < hi) rowR = __ldg(reinterpret_cast<const float4*>(a.trows) + R);
                }
                for (;;) {
                    const float bL = L >= lo ? dtL - dq : INF;       // -l on the left (dt > dq)
                    const float bR = R < hi ? dq - dtR : INF;        // l on the right (dt <= dq)
                    const bool takeL = bL < bR;
                    const float bmin = takeL ? bL : bR;
                    const float dtc = takeL ? dtL : dtR;
                    if (bmin == INF) break;                          // window exhausted (theta may be +inf)
                    if (!ti_keep(bmin, theta, dq + dtc, a.eta)) break;  // both sides beyond theta
                    const int jc = takeL ? L : R;
                    float d2;                                                   // line 15
                    if constexpr (kPre) {
                        const float4 row = takeL ? rowL : rowR;
                        if (takeL) {
                            --L;
                            if (L >= lo) {
                                dtL = __ldg(a.tdist + L);
                                rowL = __ldg(reinterpret_cast<const float4*>(a.trows) + L);
                            }
                        } else {
                            ++R;
                            if (R < hi) {
                                dtR = __ldg(a.tdist + R);
                                rowR = __ldg(reinterpret_cast<const float4*>(a.trows) + R);
                            }
                        }
                        d2 = d2_acc4(0.f, q[0], row);
                    } else {
                        if (takeL) {
                            --L;
                            if (L >= lo) dtL = __ldg(a.tdist + L);
                        } else {
                            ++R;
                            if (R < hi) dtR = __ldg(a.tdist + R);
                        }
                        d2 = d2q(a.trows + (int64_t)jc * a.dp);
                    }
                    ++evals;
                    if (d2 <= kth_d2) {                                         // line 16 (distance part)
                        const key_t key = make_key(d2, __ldg(a.torig + jc));
                        if (key < kth) {
                            if constexpr (SMEM) {
                                kth = stop.insert(key);
                            } else {
                                top.insert(key);
                                kth = top.kth();
                            }
                            kth_d2 = key_d2(kth);
                            theta = fminf(ub, __fsqrt_ru(kth_d2));              // line 17 (R8)
                        }
                    }
                }
            }
            const int qo = __ldg(a.qorig + qpos);
            if constexpr (SMEM) {
                for (int r = 0; r < a.k; ++r) write_result(a, qo, r, stop.get(r));
            } else {
#pragma unroll
                for (int s = 0; s < KMAX; ++s) {
                    const int r = s - (KMAX - a.k);
                    if (r >= 0) write_result(a, qo, r, top.a[s]);
                }
            }
        }
    }
    add_counter(&a.counters->evals_sparse, evals);
    add_counter(&a.counters->center_evals, cevals);
}

template <int DP, int KMAX, bool SMEM, int THREADS>
static void launch_tpq(Ctx& cx, const ScanArgs& a) {
    const size_t smem = SMEM ? sizeof(key_t) * (size_t)a.k * THREADS : 0;
    if (smem > 48 * 1024)
        cudaFuncSetAttribute(k_scan_tpq<DP, KMAX, SMEM, THREADS>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    int grid = occupancy_grid(cx, (const void*)k_scan_tpq<DP, KMAX, SMEM, THREADS>, THREADS, smem);
    k_scan_tpq<DP, KMAX, SMEM, THREADS><<<grid, THREADS, smem, cx.stream>>>(a);
}

// kNearests placement (Fig. 8, P:L587-609 re-derived for B200 in DESIGN.md):
// shared memory when k*4 <= th1 (k <= 28 on B200), registers for k <= 32
// otherwise; beyond the register budget (large k, NEXT-2) shared memory with
// fewer threads per CTA so k * 8 B per thread still fits. SKNN_TOPK=reg|smem
// overrides for ablation.
template <int DP>
static void launch_tpq_small_k(Ctx& cx, const ScanArgs& a) {
    const char* ov = getenv("SKNN_TOPK");
    const bool smem = ov ? (ov[0] == 's') : (a.k * 4 <= 114);
    if (smem) {
        launch_tpq<DP, 1, true, 256>(cx, a);
        return;
    }
    switch ((a.k + 3) / 4) {
        case 1: launch_tpq<DP, 4, false, 256>(cx, a); break;
        case 2: launch_tpq<DP, 8, false, 256>(cx, a); break;
        case 3: launch_tpq<DP, 12, false, 256>(cx, a); break;
        case 4: launch_tpq<DP, 16, false, 256>(cx, a); break;
        case 5: launch_tpq<DP, 20, false, 256>(cx, a); break;
        case 6: launch_tpq<DP, 24, false, 256>(cx, a); break;
        case 7: launch_tpq<DP, 28, false, 256>(cx, a); break;
        default: launch_tpq<DP, 32, false, 256>(cx, a); break;
    }
}

template <int DP>
void launch_tpq_dp(Ctx& cx, const ScanArgs& a) {
    if (a.k > 32 || DP == 0) {
        if (a.k <= 96) launch_tpq<DP, 1, true, 256>(cx, a);
        else if (a.k <= 384) launch_tpq<DP, 1, true, 64>(cx, a);
        else launch_tpq<DP, 1, true, 32>(cx, a);
        return;
    }
    if constexpr (DP > 0) launch_tpq_small_k<DP>(cx, a);
}
}  // namespace sknn
