// k_scan_common.cuh -- shared pieces of the level-2 scan kernels (Alg. 2,
// P:L355-375): launch arguments, the member-window binary search, the result
// write (Fig. 4 output R) and warp-aggregated counters.
#pragma once

#include <cuda_runtime.h>
#include <stdint.h>

#include "sknn_internal.cuh"
#include "sknn_launch.h"

namespace sknn {

struct ScanArgs {
    const float* qrows;
    const int32_t* qorig;
    const int32_t* qoff;
    const float* trows;
    const float* tdist;
    const int32_t* torig;
    const int32_t* toff;
    const float* tcent;
    const float* ub;
    const int32_t* cand;
    const int32_t* cand_count;
    const float* cand_D;
    const float* qdist;   // query's own member distance d(q, c_q)
    const float* trad;    // target cluster radius
    const int4* tinfo;    // target cluster summary {lo, hi, radius bits, smallest member distance bits}
    const int4* tiles;       // tasks {query cluster, first member, split | nsplit << 8, part}
    const int* ntiles;
    key_t* part;             // partial lists of split tasks [part][k][32]
    unsigned* theta2;        // [nq] shared k-th distance^2 bound of split queries (float bits)
    int* tile_counter;     // dynamic tile scheduler (zeroed by k_make_tiles)
    const key_t* init_topk;  // optional [nq_perm x k] keys from the dense-tile pass (NULL = none)
    const int32_t* dcount;   // optional [mq] dense pairs per query cluster (init_topk valid iff > 0)
    int mt;
    int dp;
    int k;
    int tile;
    float eta;
    int out_squared;
    long long index_base;
    int32_t* out_idx;
    float* out_dist;
    Counters* counters;
    int* probe_warps;  // non-NULL: launchers only report resident warps (no launch)
    int q_global;      // runtime-dp kernels: 1 = query rows read from global memory (too large to stage)
};

// First member position in [lo, hi) that is NOT in Alg. 2's `continue`
// region (l = dq - dt < -theta, line 12); dt descends along the array.
__device__ __forceinline__ int window_start(const float* __restrict__ tdist, int lo, int hi, float dq, float theta,
                                            float eta) {
    while (lo < hi) {
        int mid = (lo + hi) >> 1;
        float dt = __ldg(tdist + mid);
        if (!ti_keep(dt - dq, theta, dq + dt, eta)) lo = mid + 1;
        else hi = mid;
    }
    return lo;
}

// First position in [lo, hi) whose member distance dt <= dq (members are
// sorted by distance descending): the split point of the bidirectional scan.
__device__ __forceinline__ int window_start_geq(const float* __restrict__ tdist, int lo, int hi, float dq) {
    while (lo < hi) {
        int mid = (lo + hi) >> 1;
        if (__ldg(tdist + mid) > dq) lo = mid + 1;
        else hi = mid;
    }
    return lo;
}

// First position in [lo, hi) where Alg. 2 breaks (l = dq - dt > theta,
// line 10): l grows along the distance-descending member array.
__device__ __forceinline__ int window_end(const float* __restrict__ tdist, int lo, int hi, float dq, float theta,
                                          float eta) {
    while (lo < hi) {
        int mid = (lo + hi) >> 1;
        float dt = __ldg(tdist + mid);
        if (ti_keep(dq - dt, theta, dq + dt, eta)) lo = mid + 1;
        else hi = mid;
    }
    return lo;
}

__device__ __forceinline__ void write_result(const ScanArgs& a, int qorig, int r, key_t key) {
    int64_t o = (int64_t)qorig * a.k + r;
    float d2 = key_d2(key);
    a.out_dist[o] = a.out_squared ? d2 : __fsqrt_rn(d2);
    // a placeholder (fewer than k targets under an external bound, target-sharded
    // mode) gets index -1; the merge never selects it over a real key
    if (a.out_idx) a.out_idx[o] = key == kInfKey ? -1 : (int32_t)(key_idx(key) + a.index_base);
}

// warp-aggregated counter: one atomic per warp (all 32 lanes must call)
__device__ __forceinline__ void add_counter(unsigned long long* c, unsigned long long v) {
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    if ((threadIdx.x & 31) == 0 && v) atomicAdd(c, v);
}

// dispatch helpers (k_scan_tpq_dp*.cu)
template <int DP>
void launch_tpq_dp(Ctx& cx, const ScanArgs& a);

int occupancy_grid(Ctx& cx, const void* fn, int threads, size_t smem);

// k_scan_bigk.cu: warp-per-query scan for k > 32
void launch_scan_bigk(Ctx& cx, const ScanArgs& a, int dp);

}  // namespace sknn
