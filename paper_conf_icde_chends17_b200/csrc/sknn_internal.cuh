// sknn_internal.cuh -- shared device helpers and internal host structures of
// the B200-native Sweet KNN library (libsweetknn.so). Not part of the ABI.
//
// Citations: P:L<n> = PAPER.md line n (Chen, Ding, Shen, ICDE 2017).
#pragma once

#include <cuda_runtime.h>
#include <stdint.h>

#include <string>

#include "../../include/sknn.h"

namespace sknn {

constexpr int kWarp = 32;
constexpr int kMaxClusters = 8192;  // clamp of detLmNum: level-1 keeps a row of D in smem

// ------------------------------------------------------------------ keys --
// A neighbour candidate is the 64-bit key (d2 bits << 32) | target index.
// d2 >= 0, so its IEEE bits order like the value and keys order
// lexicographically by (d2, index): ties go to the lowest index (reading R2).
// Signed so that -1 can serve as an always-smaller placeholder.
typedef long long key_t;
constexpr key_t kInfKey = (key_t(0x7f800000) << 32) | key_t(0x7fffffff);
constexpr key_t kNegKey = -1;

__device__ __forceinline__ key_t make_key(float d2, int idx) {
    return (key_t(__float_as_uint(d2)) << 32) | key_t(uint32_t(idx));
}
// a < b for keys of which `a` is >= 0 (a real key or kInfKey) and `b` is a
// key or the placeholder kNegKey. Read as IEEE doubles, keys >= 0 are finite
// and non-negative (their top 11 bits are the float d2's bits 30..20, never all
// ones for a finite or +inf d2) and order exactly like the integers, and -1 is
// a NaN, so `a < -1` is false as for the integers: one DSETP (fp64 pipe)
// instead of the 64-bit integer compare pair on the ALU pipe.
// (SKNN_KEYCMP_INT builds the integer compare, for A/B timing.)
__device__ __forceinline__ bool key_lt(key_t a, key_t b) {
#ifdef SKNN_KEYCMP_INT
    return a < b;
#else
    return __longlong_as_double(a) < __longlong_as_double(b);
#endif
}
__device__ __forceinline__ float key_d2(key_t k) { return __uint_as_float(uint32_t(uint64_t(k) >> 32)); }
__device__ __forceinline__ int key_idx(key_t k) { return int(uint32_t(uint64_t(k) & 0xffffffffu)); }

// ------------------------------------------------------------- distances --
// Squared Euclidean distance in fp32, dimensions in ascending order, one
// fused multiply-add per dimension: s = fma(q_c - t_c, q_c - t_c, s).
// Zero padding columns add exactly 0. Every path (brute, sparse scan, dense
// recompute, assignment) uses these so a pair always gets the same bits.
__device__ __forceinline__ float d2_acc4(float s, float4 a, float4 b) {
    float x;
    x = a.x - b.x; s = __fmaf_rn(x, x, s);
    x = a.y - b.y; s = __fmaf_rn(x, x, s);
    x = a.z - b.z; s = __fmaf_rn(x, x, s);
    x = a.w - b.w; s = __fmaf_rn(x, x, s);
    return s;
}

// rows padded to dp (multiple of 4), 16-byte aligned
__device__ __forceinline__ float d2_rows(const float* __restrict__ a, const float* __restrict__ b, int dp) {
    const float4* a4 = reinterpret_cast<const float4*>(a);
    const float4* b4 = reinterpret_cast<const float4*>(b);
    float s = 0.f;
#pragma unroll 8
    for (int c = 0; c < dp / 4; ++c) s = d2_acc4(s, a4[c], __ldg(b4 + c));
    return s;
}

template <int DP>
__device__ __forceinline__ float d2_reg(const float4 (&q)[DP / 4], const float* __restrict__ t) {
    const float4* t4 = reinterpret_cast<const float4*>(t);
    // all row loads first (memory-level parallelism), then the fixed-order sum
    float4 r[DP / 4];
#pragma unroll
    for (int c = 0; c < DP / 4; ++c) r[c] = __ldg(t4 + c);
    float s = 0.f;
#pragma unroll
    for (int c = 0; c < DP / 4; ++c) s = d2_acc4(s, q[c], r[c]);
    return s;
}

// Fixed-point accumulation of a row into int64 sums (Lloyd update): integer
// atomics commute, so the centers do not depend on the order of the adds.
__device__ __forceinline__ void fx_accumulate(long long* dst, const float* x, int dp, double scale) {
    for (int c = 0; c < dp; ++c)
        atomicAdd(reinterpret_cast<unsigned long long*>(dst + c), (unsigned long long)__double2ll_rn((double)x[c] * scale));
}

// ------------------------------------------------------- rounding slack --
// Reading R7: every TI prune test keeps a pair unless its lower bound exceeds
// theta by more than eta * (sum of the magnitudes involved), eta = (d+8)*2^-24
// (computed distances carry a relative error of about (d+4)/2 ulps).
__device__ __forceinline__ bool ti_keep(float lb, float theta, float mag, float eta) {
    return lb <= theta + eta * (mag + theta);
}

// ------------------------------------------------------------ min trees --
// sm_100 has a three-input float minimum (FMNMX3): a min over N values takes
// about N/2 instructions instead of N - 1. min is exact and order-free, so
// the result is the same value as any fminf chain (no NaNs reach these).
__device__ __forceinline__ float fmin3(float a, float b, float c) {
    float r;
    asm("min.f32 %0, %1, %2, %3;" : "=f"(r) : "f"(a), "f"(b), "f"(c));
    return r;
}
template <int N>
__device__ __forceinline__ float min_tree(const float (&v)[N]) {
    static_assert(N == 16 || N == 32, "min_tree: 16 or 32 values");
    if constexpr (N == 32) {
        float t[11];
#pragma unroll
        for (int j = 0; j < 10; ++j) t[j] = fmin3(v[3 * j], v[3 * j + 1], v[3 * j + 2]);
        t[10] = fminf(v[30], v[31]);
        const float u0 = fmin3(t[0], t[1], t[2]), u1 = fmin3(t[3], t[4], t[5]), u2 = fmin3(t[6], t[7], t[8]);
        return fmin3(u0, u1, fmin3(u2, t[9], t[10]));
    } else {
        float t[6];
#pragma unroll
        for (int j = 0; j < 5; ++j) t[j] = fmin3(v[3 * j], v[3 * j + 1], v[3 * j + 2]);
        t[5] = v[15];
        return fmin3(fmin3(t[0], t[1], t[2]), fmin3(t[3], t[4], t[5]), t[5]);
    }
}

// ---------------------------------------------------- register top-k -----
// Sorted ascending array of KMAX keys held in registers (Fig. 8 / P:L629:
// k*4 bytes <= th2 puts kNearests in registers). Slots [0, KMAX-k) hold the
// placeholder -1 (never displaced), slots [KMAX-k, KMAX) the k best keys;
// a[KMAX-1] is the current k-th key.
template <int KMAX>
struct RegTopK {
    key_t a[KMAX];
    __device__ __forceinline__ void init(int k) {
#pragma unroll
        for (int i = 0; i < KMAX; ++i) a[i] = (i < KMAX - k) ? kNegKey : kInfKey;
    }
    __device__ __forceinline__ key_t kth() const { return a[KMAX - 1]; }
    // precondition: key < a[KMAX-1]. The comparisons c[i] = key < a[i] are
    // evaluated once (a monotone mask), then every slot is one select chain:
    // a[i] = c[i-1] ? a[i-1] : (c[i] ? key : a[i]).
    __device__ __forceinline__ void insert(key_t key) {
        bool c[KMAX];
#pragma unroll
        for (int i = 0; i < KMAX; ++i) c[i] = key_lt(key, a[i]);
#pragma unroll
        for (int i = KMAX - 1; i > 0; --i) a[i] = c[i - 1] ? a[i - 1] : (c[i] ? key : a[i]);
        a[0] = c[0] ? key : a[0];
    }
};

// ------------------------------------------------------ warp top-k -------
// Lane-distributed sorted list: lane i holds rank i of 32 slots; lanes
// [0, 32-k) hold the placeholder -1; lane 31 holds the k-th key. The warp
// analogue of the paper's per-thread heaps merged at the end.
__device__ __forceinline__ key_t warp_insert(key_t mine, key_t key, int lane) {
    key_t up = __shfl_up_sync(0xffffffffu, mine, 1);
    if (key_lt(key, mine)) mine = (lane > 0 && key_lt(key, up)) ? up : key;
    return mine;
}

__device__ __forceinline__ unsigned lane_id() { return threadIdx.x & 31u; }

}  // namespace sknn

// ------------------------------------------------------ host structures --
namespace sknn {

// One clustered point set (Step 1).
struct Side {
    int64_t n = 0;
    int d = 0, dp = 0, m = 0;
    float* rows = nullptr;     // [n x dp] permuted into cluster order, zero padded
    float* dist = nullptr;     // [n] distance to own center; descending within a cluster (R11)
    int32_t* orig = nullptr;   // [n] original row index of each permuted point
    int32_t* off = nullptr;    // [m+1] cluster offsets
    float* centers = nullptr;  // [m x dp]
    float* radius = nullptr;   // [m] max member distance (0 if empty)
    int4* tinfo = nullptr;     // [m] {lo, hi, radius bits, smallest member distance bits (+inf if empty)}:
                               // one 16-byte load per candidate cluster in level-1 and the scan
    bool owned = false;
};

struct Counters {  // device-side counters (sknn_stats)
    unsigned long long evals_sparse, evals_dense, evals_brute, center_evals, cand_pairs, dense_pairs, dist_recompute,
        topk_inserts, rows_loaded, dense_terms;
};

}  // namespace sknn

struct sknn_index {
    int device = -1;
    const void* user_ptr = nullptr;
    sknn::Side t;
    sknn_options opt;
};
