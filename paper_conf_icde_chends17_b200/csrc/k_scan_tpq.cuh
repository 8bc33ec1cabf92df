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

// kNearests of one query (Alg. 2 line 4), three placements (Fig. 8,
// P:L587-609, re-derived for B200 in DESIGN.md):
//  LIST_REG    sorted keys in registers (k*4 B <= th2); branch-free insertion
//  LIST_SORTED sorted keys in shared memory (k*4 B <= th1 = 114 B), laid out
//              like the paper's Layout 2 (Fig. 6b): slot r of thread t
//              at [r][t], so a warp's accesses to one slot are contiguous; an
//              insertion shifts only the slots above the insertion point
//  LIST_HEAP   max-heap in shared memory, same layout: the root is the k-th
//              key, an insertion is one sift-down (log2 k levels instead of
//              up to k shifts); heap-sorted once at the end
// All three keep the k smallest (d2, index) keys seen; insert() requires
// key < kth() and returns the new k-th key.
// (measured and rejected: a 4-ary heap -- log4 k dependent levels instead of
// log2 k -- C2 0.411 vs 0.411 ms, C5 52.2 vs 51.2 ms)
enum { LIST_REG = 0, LIST_SORTED = 1, LIST_HEAP = 2 };


template <int LIST, int KMAX, int STRIDE>
struct TopList;

template <int KMAX, int STRIDE>
struct TopList<LIST_REG, KMAX, STRIDE> {
    RegTopK<KMAX> r;
    int k;
    __device__ __forceinline__ void init(key_t*, int k_) {
        k = k_;
        r.init(k_);
    }
    __device__ __forceinline__ key_t kth() const { return r.kth(); }
    __device__ __forceinline__ void load_sorted(const key_t* src) {
#pragma unroll
        for (int s = 0; s < KMAX; ++s) {
            const int i = s - (KMAX - k);
            if (i >= 0) r.a[s] = src[i];
        }
    }
    __device__ __forceinline__ key_t insert(key_t key) {
        r.insert(key);
        return r.kth();
    }
    __device__ __forceinline__ void finalize() {}
    template <class F>
    __device__ __forceinline__ void emit(F f) const {
#pragma unroll
        for (int s = 0; s < KMAX; ++s) {
            const int i = s - (KMAX - k);
            if (i >= 0) f(i, r.a[s]);
        }
    }
};

template <int KMAX, int STRIDE>
struct TopList<LIST_SORTED, KMAX, STRIDE> {
    key_t* s;
    int k;
    int nfill;  // slots >= nfill still hold +inf keys: the shift starts at min(nfill, k - 1)
    __device__ __forceinline__ void init(key_t* col, int k_) {
        s = col;
        k = k_;
        nfill = 0;
        for (int r = 0; r < k; ++r) s[r * STRIDE] = kInfKey;
    }
    __device__ __forceinline__ key_t kth() const { return s[(k - 1) * STRIDE]; }
    __device__ __forceinline__ void load_sorted(const key_t* src) {
        for (int r = 0; r < k; ++r) s[r * STRIDE] = src[r];
        nfill = k;
    }
    __device__ __forceinline__ key_t insert(key_t key) {
        int i = min(nfill, k - 1);
        ++nfill;
        while (i > 0) {
            const key_t v = s[(i - 1) * STRIDE];
            if (!(key < v)) break;
            s[i * STRIDE] = v;
            --i;
        }
        s[i * STRIDE] = key;
        return s[(k - 1) * STRIDE];
    }
    __device__ __forceinline__ void finalize() {}
    template <class F>
    __device__ __forceinline__ void emit(F f) const {
        for (int r = 0; r < k; ++r) f(r, s[r * STRIDE]);
    }
};

template <int KMAX, int STRIDE>
struct TopList<LIST_HEAP, KMAX, STRIDE> {
    key_t* s;
    int k;
    __device__ __forceinline__ void init(key_t* col, int k_) {
        s = col;
        k = k_;
        for (int r = 0; r < k; ++r) s[r * STRIDE] = kInfKey;
    }
    __device__ __forceinline__ key_t kth() const { return s[0]; }
    // an ascending list read backwards is a max-heap
    __device__ __forceinline__ void load_sorted(const key_t* src) {
        for (int r = 0; r < k; ++r) s[r * STRIDE] = src[k - 1 - r];
    }
    // place `key` at the root of the heap s[0, n) and sift it down
    // (measured: pushing with a sift-up, or appending + one Floyd heapify,
    // while the list fills is no faster on C2/C3 than this full-depth
    // sift-down from the +inf root)
    __device__ __forceinline__ void sift(key_t key, int n) {
        int i = 0;
        for (;;) {
            const int l = 2 * i + 1;
            if (l >= n) break;
            key_t c = s[l * STRIDE];
            int ci = l;
            if (l + 1 < n) {
                const key_t c2 = s[(l + 1) * STRIDE];
                if (key_lt(c, c2)) {
                    c = c2;
                    ci = l + 1;
                }
            }
            if (!key_lt(key, c)) break;
            s[i * STRIDE] = c;
            i = ci;
        }
        s[i * STRIDE] = key;
    }
    // KMAX > 1: k == KMAX is a compile-time constant and the root sift is
    // fully unrolled: floor(log2 k) levels, bounds checks only on the last
    static constexpr int steps() {
        int L = 0;
        while ((2 << L) <= KMAX) ++L;
        return L;
    }
    __device__ __forceinline__ void sift_root_const(key_t key) {
        constexpr int N = KMAX, STEPS = steps();
        int i = 0;
#pragma unroll
        for (int lev = 0; lev < STEPS; ++lev) {
            const int l = 2 * i + 1;
            const bool last = lev == STEPS - 1;  // only the last level can run past the heap end
            if (last && l >= N) break;
            key_t c = s[l * STRIDE];
            int ci = l;
            if (!last || l + 1 < N) {
                const key_t c2 = s[(l + 1) * STRIDE];
                if (key_lt(c, c2)) {
                    c = c2;
                    ci = l + 1;
                }
            }
            if (!key_lt(key, c)) break;
            s[i * STRIDE] = c;
            i = ci;
        }
        s[i * STRIDE] = key;
    }
    __device__ __forceinline__ key_t insert(key_t key) {
        if constexpr (KMAX > 1) sift_root_const(key);  // the old root (the k-th key) is dropped
        else sift(key, k);
        return s[0];
    }
    // in-place heapsort: ascending order in s[0, k)
    __device__ __forceinline__ void finalize() {
        for (int end = k - 1; end > 0; --end) {
            const key_t top = s[0];
            const key_t last = s[end * STRIDE];
            s[end * STRIDE] = top;
            sift(last, end);
        }
    }
    template <class F>
    __device__ __forceinline__ void emit(F f) const {
        for (int r = 0; r < k; ++r) f(r, s[r * STRIDE]);
    }
};

// One warp tile of the thread-per-query scan (Alg. 2 for 32 queries).
template <int DP, int KMAX, int LIST, int THREADS, bool SPLIT>
__device__ __forceinline__ void tpq_tile(const ScanArgs& a, const int4 tl, key_t* s_topk, unsigned long long& evals,
                                         unsigned long long& cevals, unsigned long long& ins,
                                         unsigned long long& rows) {
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
    TopList<LIST, KMAX, THREADS> top;
    top.init(s_topk + threadIdx.x, a.k);
    key_t kth = top.kth();
    const float ub = a.ub[qc];
    float theta = ub;
    // no member beyond UB can enter the list (UB bounds every query's k-th
    // distance, R7), so inserts are gated by ub^2 until the list is full
    float kth_d2 = __fmul_ru(ub, ub);
    if (a.init_topk && a.dcount[qc] > 0) {  // continue from the dense-tile pass
        if (split == 0) {  // (the other tasks of a split tile only take its bound)
            top.load_sorted(a.init_topk + (int64_t)qpos * a.k);
            kth = top.kth();
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
            const int4 ti = __ldg(a.tinfo + tc);  // {lo, hi, r_t, smallest member distance}
            const float D = __ldg(cD + c), rt = __int_as_float(ti.z);
            if (!ti_keep(D - rown - rt, theta, D + rown + rt, a.eta)) continue;
            const int lo = ti.x, hi = ti.y;
            const float dq = __fsqrt_rn(d2q(a.tcent + (int64_t)tc * a.dp));  // Alg. 2 line 6
            ++cevals;
            // empty window: every member distance lies in [dt_min, r_t]
            if (!ti_keep(dq - rt, theta, dq + rt, a.eta)) continue;
            const float dtmin = __int_as_float(ti.w);
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
                    if (key_lt(key, kth)) {
                        ++ins;
                        kth = top.insert(key);
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
                ++rows;
                consider(d2, jc);
            }
        }
        if (SPLIT) {  // partial list of this task -> k_merge_split
            key_t* pl = a.part + (int64_t)tl.w * a.k * 32 + lane;
            top.finalize();
            top.emit([&](int r, key_t v) { pl[r * 32] = v; });
        } else {
            const int qo = __ldg(a.qorig + qpos);
            top.finalize();
            top.emit([&](int r, key_t v) { write_result(a, qo, r, v); });
        }
    }
}

// Members evaluated per block of the warp-union walk (rows held in registers
// while their distances are computed): ~32 floats of row data per block.
#ifndef SKNN_U4
#define SKNN_U4 8
#endif
#ifndef SKNN_COLLECT
#define SKNN_COLLECT 1
#endif
#ifndef SKNN_MINFIRST
#define SKNN_MINFIRST 1
#endif
#ifndef SKNN_U16
#define SKNN_U16 2
#endif
#ifndef SKNN_MINB16
#define SKNN_MINB16 1
#endif
#ifndef SKNN_UNION_MINB4
#define SKNN_UNION_MINB4 3
#endif
#ifndef SKNN_AB4
#define SKNN_AB4 2
#endif
#ifndef SKNN_AB16
#define SKNN_AB16 1
#endif
// blocks of union_block<DP>() members per alive test of the walk (overshoot
// past a side's last needed member: at most U * AB - 1 extra evaluations)
template <int DP>
constexpr int union_alive_blocks() {
    return DP == 0 ? 1 : (DP <= 4 ? SKNN_AB4 : (DP <= 16 && DP > 8 ? SKNN_AB16 : 1));
}
template <int DP>
constexpr int union_block() {
    return DP == 0 ? 1 : (DP <= 4 ? SKNN_U4 : (DP <= 8 ? 4 : (DP <= 16 ? SKNN_U16 : 1)));
}

// One warp tile of the thread-per-query scan with a WARP-UNION member walk
// (the regularity side of Sweet KNN's reconciliation, §IV, on B200): for a
// candidate cluster the 32 lanes walk the union of their Alg. 2 windows
// together, every lane computing the distance of the same member, so each row
// is one broadcast load for the whole warp and the loop has no per-lane
// control flow except the kNearests insert. The walk starts at the split
// point of a middle lane's dq and grows both sides in blocks of
// union_block<DP>() members; a side stops when no lane's window (Alg. 2
// lines 10-13 with its own running theta) reaches its next member. Lanes
// evaluate members outside their own window (harmless: every evaluated
// distance is a real (query, target) distance and the list keeps the k
// smallest keys), so every member of every lane's window is evaluated
// (monotone break tests, DESIGN.md §2 exactness argument).
template <int DP, int KMAX, int LIST, int THREADS, bool SPLIT, int BUF>
__device__ __forceinline__ void union_tile(const ScanArgs& a, const int4 tl, key_t* s_topk, unsigned long long& evals,
                                           unsigned long long& cevals, unsigned long long& ins,
                                         unsigned long long& rows) {
    constexpr unsigned FULL = 0xffffffffu;
    const int lane = threadIdx.x & 31;
    const int qc = tl.x;
    const int qlo = a.qoff[qc], qsz = a.qoff[qc + 1] - qlo;
    const int i = tl.y + lane;
    const bool active = i < qsz;
    const int qpos = qlo + (active ? i : 0);  // an idle lane shadows the tile's first query
    const int split = SPLIT ? (tl.z & 0xff) : 0;
    const int nsplit = SPLIT ? (tl.z >> 8) : 1;
    constexpr int QV = DP > 0 ? DP / 4 : 1;
    constexpr int U = union_block<DP>();
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
    TopList<LIST, KMAX, THREADS> top;
    top.init(s_topk + threadIdx.x, a.k);
    key_t kth = top.kth();
    const float ub = a.ub[qc];
    float theta = ub;
    float kth_d2 = __fmul_ru(ub, ub);
    if (a.init_topk && a.dcount[qc] > 0) {  // continue from the dense-tile pass
        if (split == 0) {
            top.load_sorted(a.init_topk + (int64_t)qpos * a.k);
            kth = top.kth();
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
    const float4* trow4 = reinterpret_cast<const float4*>(a.trows);
    bool dirty = false;
    // BUF > 0: keys that pass the (possibly stale) k-th bound wait in a
    // per-lane register buffer; the warp flushes all buffers into the lists
    // together once some lane's buffer is full, so the insert code runs with
    // many lanes active instead of once per member with a few
    key_t buf[BUF > 0 ? BUF : 1];
    int nb = 0;
    auto flush = [&]() {
#pragma unroll
        for (int b = 0; b < BUF; ++b) {
            if (b < nb && key_lt(buf[b], kth)) {
                ++ins;
                kth = top.insert(buf[b]);
            }
        }
        nb = 0;
        if (key_d2(kth) < kth_d2) {
            kth_d2 = key_d2(kth);
            dirty = true;
        }
    };
    auto consider = [&](float d2, int jc) {  // called by all 32 lanes
        if (active && d2 <= kth_d2) {                                // Alg. 2 line 16 (distance part)
            const key_t key = make_key(d2, __ldg(a.torig + jc));
            if (key_lt(key, kth)) {
                if constexpr (BUF > 0) {
#pragma unroll
                    for (int b = 0; b < BUF; ++b)
                        if (b == nb) buf[b] = key;
                    ++nb;
                } else {
                    ++ins;
                    kth = top.insert(key);
                    if (key_d2(kth) < kth_d2) {
                        kth_d2 = key_d2(kth);
                        dirty = true;  // theta follows once per block
                    }
                }
            }
        }
        if constexpr (BUF > 0) {
            if (__any_sync(FULL, nb == BUF)) flush();
        }
    };
    // line 17 (R8): theta = min(UB, sqrt(k-th d2) rounded up), refreshed once
    // per block of members (a stale, larger theta only evaluates more)
    auto refresh = [&]() {
        if (dirty) {
            dirty = false;
            theta = fminf(ub, __fsqrt_ru(kth_d2));
            if (SPLIT && active) atomicMin(th2, __float_as_uint(kth_d2));
        }
    };
    // distances of members j0, j0 + step, ... (n of them, n <= U): all row
    // loads first (one broadcast transaction each), then the fixed-order sums
    auto eval_block = [&](int j0, int step, int n) {
        if constexpr (DP > 0) {
            float4 r[U][DP / 4];
#pragma unroll
            for (int u = 0; u < U; ++u) {
                const int j = j0 + step * min(u, n - 1);
#pragma unroll
                for (int c = 0; c < DP / 4; ++c) r[u][c] = __ldg(trow4 + (int64_t)j * (DP / 4) + c);
            }
#if SKNN_COLLECT
            if constexpr (BUF == 0) {
                // all U distances first; the members that pass the lane's
                // current k-th bound are collected in a bit mask and inserted
                // by a per-lane loop, so the insert code runs once per
                // max-over-lanes pending count with every pending lane active
                // (instead of once per member that any lane inserts)
                float dd[U];
                unsigned pass = 0;
#pragma unroll
                for (int u = 0; u < U; ++u) {
                    float s = 0.f;
#pragma unroll
                    for (int c = 0; c < DP / 4; ++c) s = d2_acc4(s, q[c], r[u][c]);
                    dd[u] = s;
                }
#if SKNN_MINFIRST
                // one compare of the block minimum first (members past n repeat the
                // last member, so the minimum is still a real distance of the block)
                float mn = dd[0];
#pragma unroll
                for (int u = 1; u < U; u += 2) mn = (u + 1 < U) ? fmin3(mn, dd[u], dd[u + 1]) : fminf(mn, dd[u]);
                if (active && mn <= kth_d2)
#endif
                {
#pragma unroll
                    for (int u = 0; u < U; ++u)
                        // Alg. 2 line 16 (distance part); a lane past the tile's last
                        // query only shadows the walk and never inserts
                        if (active && u < n && dd[u] <= kth_d2) pass |= 1u << u;
                }
                while (pass) {
                    const int u = __ffs(pass) - 1;
                    pass &= pass - 1;
                    float d2 = dd[0];
#pragma unroll
                    for (int v = 1; v < U; ++v)
                        if (u == v) d2 = dd[v];
                    if (d2 <= kth_d2) {  // re-checked: an earlier insert may have lowered the bound
                        const key_t key = make_key(d2, __ldg(a.torig + j0 + step * u));
                        if (key_lt(key, kth)) {
                            ++ins;
                            kth = top.insert(key);
                            if (key_d2(kth) < kth_d2) {
                                kth_d2 = key_d2(kth);
                                dirty = true;
                            }
                        }
                    }
                }
                return;
            }
#endif
#pragma unroll
            for (int u = 0; u < U; ++u) {
                if (u < n) {
                    float s = 0.f;
#pragma unroll
                    for (int c = 0; c < DP / 4; ++c) s = d2_acc4(s, q[c], r[u][c]);
                    consider(s, j0 + step * u);
                }
            }
        } else {
            for (int u = 0; u < n; ++u) consider(d2_rows(qrow, a.trows + (int64_t)(j0 + step * u) * a.dp, a.dp),
                                                 j0 + step * u);
        }
    };
    for (int c = split; c < ncand; c += nsplit) {  // warp-uniform: the tile's lanes share qc
        if (SPLIT) {  // the bound the tile's other tasks have reached
            const float g = __uint_as_float(*(volatile unsigned*)th2);
            if (g < kth_d2) {
                kth_d2 = g;
                theta = fminf(ub, __fsqrt_ru(g));
            }
        }
        const int tc = __ldg(cl + c);
        // per-query 2-landmark bound (Eq. 3 with the query in place of the
        // query cluster's farthest member): D - d(q,c_q) - r_t <= d(q,t)
        const int4 ti = __ldg(a.tinfo + tc);  // {lo, hi, r_t, smallest member distance}
        const float D = __ldg(cD + c), rt = __int_as_float(ti.z);
        bool ok = active && ti_keep(D - rown - rt, theta, D + rown + rt, a.eta);
        if (!__any_sync(FULL, ok)) continue;
        const int lo = ti.x, hi = ti.y;
        const float dq = __fsqrt_rn(d2q(a.tcent + (int64_t)tc * a.dp));  // Alg. 2 line 6
        cevals += active;
        // empty window: every member distance lies in [dt_min, r_t]
        const float dtmin = __int_as_float(ti.w);
        ok = ok && ti_keep(dq - rt, theta, dq + rt, a.eta) && ti_keep(dtmin - dq, theta, dq + dtmin, a.eta);
        const unsigned okm = __ballot_sync(FULL, ok);
        if (!okm) continue;
        // split point at the dq of the lane midway between the first and last
        // lane with a window (any split point is correct; lanes of a tile are
        // in member-distance order, so this is near their median)
        const int mid = ((__ffs(okm) - 1) + (31 - __clz(okm))) >> 1;
        const float dsplit = __shfl_sync(FULL, dq, mid);
        const int p = window_start_geq(a.tdist, lo, hi, dsplit);  // first member with dt <= dsplit
        int R = p, L = p - 1;
        // right side (dt <= dsplit, l = dq - dt growing): lane needs member R
        // unless Alg. 2 breaks there (line 10); left side (dt > dsplit): lane
        // needs member L unless it is in the `continue` region (line 12)
        bool aliveR = R < hi && __any_sync(FULL, ok && ti_keep(dq - __ldg(a.tdist + R), theta,
                                                                dq + __ldg(a.tdist + R), a.eta));
        bool aliveL = L >= lo && __any_sync(FULL, ok && ti_keep(__ldg(a.tdist + L) - dq, theta,
                                                                 dq + __ldg(a.tdist + L), a.eta));
        unsigned walked = 0;
        // the alive test (a load of the next member distance + a vote) runs once
        // per UA = U * AB members; the block is evaluated U members at a time
        constexpr int AB = union_alive_blocks<DP>();
        while (aliveR || aliveL) {
            if (aliveR) {
                const int n = min(U * AB, hi - R);
#pragma unroll
                for (int sb = 0; sb < AB; ++sb)
                    if (sb * U < n) eval_block(R + sb * U, 1, min(U, n - sb * U));
                refresh();
                R += n;
                walked += n;
                float dtn = 0.f;
                if (R < hi) dtn = __ldg(a.tdist + R);
                aliveR = R < hi && __any_sync(FULL, ok && ti_keep(dq - dtn, theta, dq + dtn, a.eta));
            }
            if (aliveL) {
                const int n = min(U * AB, L - lo + 1);
#pragma unroll
                for (int sb = 0; sb < AB; ++sb)
                    if (sb * U < n) eval_block(L - sb * U, -1, min(U, n - sb * U));
                refresh();
                L -= n;
                walked += n;
                float dtn = 0.f;
                if (L >= lo) dtn = __ldg(a.tdist + L);
                aliveL = L >= lo && __any_sync(FULL, ok && ti_keep(dtn - dq, theta, dq + dtn, a.eta));
            }
        }
        if (active) evals += walked;
        if (lane == 0) rows += walked;  // one broadcast row load per member for the warp
    }
    if constexpr (BUF > 0) flush();
    if (active) {
        if (SPLIT) {  // partial list of this task -> k_merge_split
            key_t* pl = a.part + (int64_t)tl.w * a.k * 32 + lane;
            top.finalize();
            top.emit([&](int r, key_t v) { pl[r * 32] = v; });
        } else {
            const int qo = __ldg(a.qorig + qpos);
            top.finalize();
            top.emit([&](int r, key_t v) { write_result(a, qo, r, v); });
        }
    }
}

// DP == 0: runtime dp (> 32), the query row is re-read from L1/L2 (large k only)
// register caps (measured): DP == 4 with a shared-memory list at 64 (4 CTAs
// / SM; C2 0.62 vs 0.68 ms at the compiler's 80), register lists at 128
// (2 CTAs / SM; the two inlined task bodies otherwise take ~190)
template <int DP, int LIST, int THREADS, int WALK>
constexpr int tpq_min_blocks() {
    return THREADS != 256 ? 1 : (LIST == LIST_REG ? 2 : (DP == 4 ? (WALK ? SKNN_UNION_MINB4 : 4) : (DP == 16 ? SKNN_MINB16 : 1)));
}
template <int DP, int KMAX, int LIST, int THREADS, int WALK>
__global__ void __launch_bounds__(THREADS, (tpq_min_blocks<DP, LIST, THREADS, WALK>())) k_scan_tpq(ScanArgs a) {
    extern __shared__ __align__(16) key_t s_topk[];  // [k][THREADS] for the shared-memory lists
    const int lane = threadIdx.x & 31;
    const int ntiles = *a.ntiles;
    unsigned long long evals = 0, cevals = 0, ins = 0, rows = 0;
    for (;;) {
        int tile = 0;
        if (lane == 0) tile = atomicAdd(a.tile_counter, 1);
        tile = __shfl_sync(0xffffffffu, tile, 0);
        if (tile >= ntiles) break;
        const int4 tl = a.tiles[tile];
        if constexpr (WALK > 0) {
            constexpr int BUF = WALK == 2 ? 4 : 0;
            if ((tl.z >> 8) > 1) union_tile<DP, KMAX, LIST, THREADS, true, BUF>(a, tl, s_topk, evals, cevals, ins, rows);
            else union_tile<DP, KMAX, LIST, THREADS, false, BUF>(a, tl, s_topk, evals, cevals, ins, rows);
        } else {
            if ((tl.z >> 8) > 1) tpq_tile<DP, KMAX, LIST, THREADS, true>(a, tl, s_topk, evals, cevals, ins, rows);
            else tpq_tile<DP, KMAX, LIST, THREADS, false>(a, tl, s_topk, evals, cevals, ins, rows);
        }
    }
    add_counter(&a.counters->evals_sparse, evals);
    add_counter(&a.counters->center_evals, cevals);
    add_counter(&a.counters->topk_inserts, ins);
    add_counter(&a.counters->rows_loaded, rows);
}

template <int DP, int KMAX, int LIST, int THREADS, int WALK>
static void launch_tpq_walk(Ctx& cx, const ScanArgs& a) {
    const size_t smem = LIST != LIST_REG ? sizeof(key_t) * (size_t)a.k * THREADS : 0;
    auto fn = k_scan_tpq<DP, KMAX, LIST, THREADS, WALK>;
    if (smem > 48 * 1024) cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    int grid = occupancy_grid(cx, (const void*)fn, THREADS, smem);
    if (a.probe_warps) {  // dry run: report resident warps for the task planner
        *a.probe_warps = grid * (THREADS / 32);
        return;
    }
    fn<<<grid, THREADS, smem, cx.stream>>>(a);
}

// member walk: warp-union with immediate inserts (k <= 24) or with buffered
// inserts (k > 24, where a heap insert is deep enough that running it for many
// lanes at once pays: C5 k=32 93.6 -> 84.5 ms; C2 k=20 0.94 -> 1.54 ms,
// C3 k=16 4.13 -> 4.24 ms the other way). SKNN_WALK=union|ubuf|lane
// (per-lane LB-ordered walk) overrides for ablation.
template <int DP, int KMAX, int LIST, int THREADS>
static void launch_tpq(Ctx& cx, const ScanArgs& a) {
    if constexpr (LIST == LIST_HEAP && KMAX > 1) {  // compile-time k: the default walk only
        launch_tpq_walk<DP, KMAX, LIST, THREADS, (KMAX > 24 ? 2 : 1)>(cx, a);
    } else {
        const char* w = getenv("SKNN_WALK");
        int walk = a.k > 24 ? 2 : 1;
        if (w) walk = w[0] == 'l' ? 0 : (w[1] == 'b' ? 2 : 1);
        if (walk == 0) launch_tpq_walk<DP, KMAX, LIST, THREADS, 0>(cx, a);
        else if (walk == 1) launch_tpq_walk<DP, KMAX, LIST, THREADS, 1>(cx, a);
        else launch_tpq_walk<DP, KMAX, LIST, THREADS, 2>(cx, a);
    }
}

// kNearests placement (Fig. 8, P:L587-609 re-derived for B200 in DESIGN.md):
// shared memory, as a max-heap, for every k. Measured with the warp-union walk
// (tools/sweep.py): C2 k=20 heap 0.49 / sorted 0.50 / registers 1.25 ms, C5
// k=32 heap 62.5 / registers 79.5 / sorted 89.4 ms. SKNN_TOPK=reg|smem|heap
// overrides for ablation.
static int topk_override() {
    const char* ov = getenv("SKNN_TOPK");
    if (!ov) return -1;
    return ov[0] == 'r' ? LIST_REG : (ov[0] == 'h' ? LIST_HEAP : LIST_SORTED);
}

template <int DP, int KMAX>
static void launch_tpq_reg(Ctx& cx, const ScanArgs& a) {
    launch_tpq<DP, KMAX, LIST_REG, 256>(cx, a);
}

template <int DP>
static void launch_tpq_small_k(Ctx& cx, const ScanArgs& a) {
    int list = topk_override();
    if (list < 0) list = LIST_HEAP;
    if (list == LIST_SORTED) {
        launch_tpq<DP, 1, LIST_SORTED, 256>(cx, a);
        return;
    }
    if (list == LIST_HEAP) {
        // the configs' k (C1 8, C3/C4 16, C2 20, C5 32) get a compile-time k
        // (unrolled sift); any other k runs the runtime-k heap
        if (!getenv("SKNN_HEAP_RT")) {
            switch (a.k) {
                case 8: launch_tpq<DP, 8, LIST_HEAP, 256>(cx, a); return;
                case 16: launch_tpq<DP, 16, LIST_HEAP, 256>(cx, a); return;
                case 20: launch_tpq<DP, 20, LIST_HEAP, 256>(cx, a); return;
                case 32: launch_tpq<DP, 32, LIST_HEAP, 256>(cx, a); return;
                default: break;
            }
        }
        launch_tpq<DP, 1, LIST_HEAP, 256>(cx, a);
        return;
    }
    switch ((a.k + 3) / 4) {
        case 1: launch_tpq_reg<DP, 4>(cx, a); break;
        case 2: launch_tpq_reg<DP, 8>(cx, a); break;
        case 3: launch_tpq_reg<DP, 12>(cx, a); break;
        case 4: launch_tpq_reg<DP, 16>(cx, a); break;
        case 5: launch_tpq_reg<DP, 20>(cx, a); break;
        case 6: launch_tpq_reg<DP, 24>(cx, a); break;
        case 7: launch_tpq_reg<DP, 28>(cx, a); break;
        default: launch_tpq_reg<DP, 32>(cx, a); break;
    }
}

// large k (NEXT-2): the list stays in shared memory (heap by default, sorted
// with SKNN_TOPK=smem) with fewer threads per CTA so k * 8 B per thread fits
template <int DP, int LIST>
static void launch_tpq_large_k(Ctx& cx, const ScanArgs& a) {
    if (a.k <= 96) launch_tpq<DP, 1, LIST, 256>(cx, a);
    else if (a.k <= 384) launch_tpq<DP, 1, LIST, 64>(cx, a);
    else launch_tpq<DP, 1, LIST, 32>(cx, a);
}

template <int DP>
void launch_tpq_dp(Ctx& cx, const ScanArgs& a) {
    if (a.k > 32 || DP == 0) {
        if (topk_override() == LIST_SORTED) launch_tpq_large_k<DP, LIST_SORTED>(cx, a);
        else launch_tpq_large_k<DP, LIST_HEAP>(cx, a);
        return;
    }
    if constexpr (DP > 0) launch_tpq_small_k<DP>(cx, a);
}
}  // namespace sknn
