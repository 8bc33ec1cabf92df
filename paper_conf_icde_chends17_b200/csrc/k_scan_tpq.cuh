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
    __device__ __forceinline__ key_t insert(key_t key) { return insert_from(key, k - 1); }
    // slots >= n are still +inf: start the shift at min(n, k - 1)
    __device__ __forceinline__ key_t insert_from(key_t key, int i) {
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

// One warp tile of the thread-per-query scan (Alg. 2 for 32 queries).
template <int DP, int KMAX, bool SMEM, int THREADS, bool SPLIT>
__device__ __forceinline__ void tpq_tile(const ScanArgs& a, const int4 tl, key_t* s_topk, unsigned long long& evals,
                                         unsigned long long& cevals) {
    const float INF = __int_as_float(0x7f800000);
    const int lane = threadIdx.x & 31;
    const int qc = tl.x;
    const int qlo = a.qoff[qc], qsz = a.qoff[qc + 1] - qlo;
    const int i = tl.y + lane;
    const bool active = i < qsz;
    const int qpos = qlo + (active ? i : 0);
    // SPLIT: this task takes candidates split, split + nsplit, ... of a split
    // tile (k_make_tasks); a separate instantiation keeps the unsplit loop lean
    const int split = SPLIT ? (tl.z & 0xff) : 0;
    const int nsplit = SPLIT ? (tl.z >> 8) : 1;
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
    // slots >= nfill still hold +inf keys (the shift starts at nfill); no
    // member beyond UB can enter the list (UB bounds every query's k-th
    // distance, R7), so inserts are gated by ub^2 until the list is full
    int nfill = 0;
    float kth_d2 = __fmul_ru(ub, ub);
    if (a.init_topk && a.dcount[qc] > 0) {  // continue from the dense-tile pass
        if (split == 0) {  // (the other tasks of a split tile only take its bound)
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
            nfill = a.k;
            kth_d2 = fminf(kth_d2, key_d2(kth));
        } else {
            kth_d2 = fminf(kth_d2, key_d2(a.init_topk[(int64_t)qpos * a.k + a.k - 1]));
        }
        theta = fminf(ub, __fsqrt_ru(kth_d2));
    }
    const int ncand = a.cand_count[qc];
    const int32_t* cl = a.cand + (int64_t)qc * a.mt;
    const float* cD = a.cand_D + (int64_t)qc * a.mt;
    const float rown = __ldg(a.qdist + qpos);  // d(q, c_q)
    unsigned* th2 = a.theta2 + qpos;
    if (active) {
        for (int c = split; c < ncand; c += nsplit) {
            if (SPLIT) {  // the bound the tile's other tasks have reached
                const float g = __uint_as_float(*(volatile unsigned*)th2);
                if (g < kth_d2) {
                    kth_d2 = g;
                    theta = fminf(ub, __fsqrt_ru(g));
                }
            }
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
            auto consider = [&](float d2, int jc) {
                if (d2 <= kth_d2) {                                         // line 16 (distance part)
                    const key_t key = make_key(d2, __ldg(a.torig + jc));
                    if (key < kth) {
                        if constexpr (SMEM) {
                            kth = stop.insert_from(key, min(nfill, a.k - 1));
                            ++nfill;
                        } else {
                            top.insert(key);
                            kth = top.kth();
                        }
                        if (key_d2(kth) < kth_d2) {
                            kth_d2 = key_d2(kth);
                            theta = fminf(ub, __fsqrt_ru(kth_d2));          // line 17 (R8)
                            if (SPLIT) atomicMin(th2, __float_as_uint(kth_d2));
                        }
                    }
                }
            };
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
                consider(d2, jc);
            }
        }
        if (SPLIT) {  // partial list of this task -> k_merge_split
            key_t* pl = a.part + (int64_t)tl.w * a.k * 32 + lane;
            if constexpr (SMEM) {
                for (int r = 0; r < a.k; ++r) pl[r * 32] = stop.get(r);
            } else {
#pragma unroll
                for (int s = 0; s < KMAX; ++s) {
                    const int r = s - (KMAX - a.k);
                    if (r >= 0) pl[r * 32] = top.a[s];
                }
            }
        } else {
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
}

// DP == 0: runtime dp (> 32), the query row is re-read from L1/L2 (large k only)
// register caps (measured): DP == 4 with the shared-memory list at 64 (4 CTAs
// / SM; C2 0.62 vs 0.68 ms at the compiler's 80), register lists at 128
// (2 CTAs / SM; the two inlined task bodies otherwise take ~190)
template <int DP, bool SMEM, int THREADS>
constexpr int tpq_min_blocks() {
    return THREADS != 256 ? 1 : (!SMEM ? 2 : (DP == 4 ? 4 : 1));
}
template <int DP, int KMAX, bool SMEM, int THREADS>
__global__ void __launch_bounds__(THREADS, (tpq_min_blocks<DP, SMEM, THREADS>())) k_scan_tpq(ScanArgs a) {
    extern __shared__ __align__(16) key_t s_topk[];  // [k][256] when SMEM
    const int lane = threadIdx.x & 31;
    const int ntiles = *a.ntiles;
    unsigned long long evals = 0, cevals = 0;
    for (;;) {
        int tile = 0;
        if (lane == 0) tile = atomicAdd(a.tile_counter, 1);
        tile = __shfl_sync(0xffffffffu, tile, 0);
        if (tile >= ntiles) break;
        const int4 tl = a.tiles[tile];
        if ((tl.z >> 8) > 1) tpq_tile<DP, KMAX, SMEM, THREADS, true>(a, tl, s_topk, evals, cevals);
        else tpq_tile<DP, KMAX, SMEM, THREADS, false>(a, tl, s_topk, evals, cevals);
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
    if (a.probe_warps) {  // dry run: report resident warps for the task planner
        *a.probe_warps = grid * (THREADS / 32);
        return;
    }
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
