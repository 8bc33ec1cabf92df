// k_build.cu -- Step 1 of the method: landmark/cluster construction
// (§II-C Step 1; §III-A), re-designed for B200.
//
//   k_pad_rows         X [n x d] -> Xp [n x dp] zero padded (16-byte rows for float4 loads, Fig. 7b / P:L559)
//   k_landmark_draw    10 trials x m distinct random candidate landmarks; a keyed Feistel
//                      permutation of [0, n) gives distinct indices without a set
//   k_landmark_sums    S = sum of pairwise distances of each trial's candidates
//   k_landmark_pick    argmax_trial S (first trial on ties) and gather of the winning centers
//   k_assign<DP>       nearest center of every point, ties -> lowest center;
//                      optional Lloyd accumulation (north_star "a few Lloyd iterations", R9),
//                      cluster histogram, and the exact fp32 distance to the chosen center
//   k_lloyd_update     center = mean of members (empty cluster keeps its center)
//   k_offsets          exclusive scan of cluster counts -> CSR offsets (replaces the paper's CPU
//                      allocation between two kernels: no host round trip)
//   k_scatter_keys     one sort key per point at its cluster slot
//   k_segsort_small/big  members of every cluster sorted by distance descending, index ascending
//                      ("sorts those points in descending order", reading R11)
//   k_gather_side      permuted padded rows, member distances, original indices
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#include "sknn_internal.cuh"
#include "sknn_launch.h"

namespace sknn {

typedef unsigned long long u64;

__global__ void k_pad_rows(const float* __restrict__ X, int64_t n, int d, int dp, float* __restrict__ Xp) {
    int64_t total = n * (int64_t)dp;
    for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < total; e += (int64_t)gridDim.x * blockDim.x) {
        int64_t r = e / dp;
        int c = int(e - r * dp);
        Xp[e] = (c < d) ? X[r * d + c] : 0.f;
    }
}

// ---------------------------------------------------- landmark sampler --
__device__ __forceinline__ uint32_t mix32(uint64_t x) {
    x ^= x >> 30; x *= 0xbf58476d1ce4e5b9ull;
    x ^= x >> 27; x *= 0x94d049bb133111ebull;
    x ^= x >> 31;
    return uint32_t(x >> 16);
}

// bijection on [0, n): 4-round Feistel network on 2*half bits + cycle walking
__device__ uint32_t perm_index(uint32_t i, uint32_t n, uint64_t key) {
    int bits = 2;
    while ((1ull << bits) < n) ++bits;
    if (bits & 1) ++bits;
    int half = bits / 2;
    uint32_t mask = (1u << half) - 1u;
    uint32_t v = i;
    do {
        uint32_t L = v >> half, R = v & mask;
#pragma unroll
        for (int r = 0; r < 4; ++r) {
            uint32_t F = mix32(key * 0x9e3779b97f4a7c15ull + (uint64_t(r) << 40) + R) & mask;
            uint32_t nl = R;
            R = L ^ F;
            L = nl;
        }
        v = (L << half) | R;
    } while (v >= n);
    return v;
}

__global__ void k_landmark_draw(int64_t n, int m, int trials, uint64_t seed, int32_t* __restrict__ idx) {
    int t = blockIdx.y;
    for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < m; i += gridDim.x * blockDim.x)
        idx[t * m + i] = (int32_t)perm_index((uint32_t)i, (uint32_t)n, seed * 1315423911ull + t + 1);
}

// Pairwise-distance sum of each trial's candidate set, tiled: one
// CTA per (trial, 64x64 tile of the upper triangle of the m x m pair matrix);
// both row blocks are staged in shared memory (dp <= 128) so every distance
// reads on-chip data; fixed-order reductions keep the sum deterministic.
constexpr int kLmTile = 64;
__global__ void __launch_bounds__(256) k_landmark_sums(const float* __restrict__ Xp, int dp, int m,
                                                       const int32_t* __restrict__ idx, int nb,
                                                       double* __restrict__ partial) {
    extern __shared__ __align__(16) float s_rows[];  // [2 x 64 x dp]
    const int t = blockIdx.y;
    // linear tile -> (bi, bj), bi <= bj
    int tl = blockIdx.x, bi = 0;
    while (tl >= nb - bi) { tl -= nb - bi; ++bi; }
    const int bj = bi + tl;
    const bool smem = dp <= 128;
    float* A = s_rows;
    float* B = s_rows + kLmTile * dp;
    if (smem) {
        for (int e = threadIdx.x; e < kLmTile * dp / 4; e += blockDim.x) {
            int r = e / (dp / 4), c = e % (dp / 4);
            int ia = bi * kLmTile + r, ib = bj * kLmTile + r;
            float4 z = make_float4(0.f, 0.f, 0.f, 0.f);
            reinterpret_cast<float4*>(A)[e] = ia < m ? __ldg(reinterpret_cast<const float4*>(Xp + (int64_t)idx[t * m + ia] * dp) + c) : z;
            reinterpret_cast<float4*>(B)[e] = ib < m ? __ldg(reinterpret_cast<const float4*>(Xp + (int64_t)idx[t * m + ib] * dp) + c) : z;
        }
        __syncthreads();
    }
    double s = 0.0;
    if (smem) {
        // 16 x 16 threads, each a 4 x 4 block of pairs with its rows in registers;
        // the 16 distances sum in fp32 (MUFU sqrt) before one double add: S only
        // ranks the trials, and the fixed order keeps it deterministic
        const int ti = threadIdx.x >> 4, tj = threadIdx.x & 15;
        const float4* A4 = reinterpret_cast<const float4*>(A);
        const float4* B4 = reinterpret_cast<const float4*>(B);
        const int dq = dp / 4;
        float acc[4][4];
#pragma unroll
        for (int u = 0; u < 4; ++u)
#pragma unroll
            for (int v = 0; v < 4; ++v) acc[u][v] = 0.f;
        for (int c = 0; c < dq; ++c) {
            float4 ra[4], rb[4];
#pragma unroll
            for (int u = 0; u < 4; ++u) {
                ra[u] = A4[(ti * 4 + u) * dq + c];
                rb[u] = B4[(tj * 4 + u) * dq + c];
            }
#pragma unroll
            for (int u = 0; u < 4; ++u)
#pragma unroll
                for (int v = 0; v < 4; ++v) acc[u][v] = d2_acc4(acc[u][v], ra[u], rb[v]);
        }
        float fs = 0.f;
#pragma unroll
        for (int u = 0; u < 4; ++u)
#pragma unroll
            for (int v = 0; v < 4; ++v) {
                const int gi = bi * kLmTile + ti * 4 + u, gj = bj * kLmTile + tj * 4 + v;
                float r;
                asm("sqrt.approx.ftz.f32 %0, %1;" : "=f"(r) : "f"(acc[u][v]));
                fs += (gi < gj && gj < m) ? r : 0.f;
            }
        s = (double)fs;
    } else {
        for (int p = threadIdx.x; p < kLmTile * kLmTile; p += blockDim.x) {
            int i = p / kLmTile, j = p % kLmTile;
            int gi = bi * kLmTile + i, gj = bj * kLmTile + j;
            if (gi >= gj || gj >= m) continue;
            const float* ra = Xp + (int64_t)idx[t * m + gi] * dp;
            const float* rb = Xp + (int64_t)idx[t * m + gj] * dp;
            float d2 = 0.f;
            for (int c = 0; c < dp / 4; ++c)
                d2 = d2_acc4(d2, reinterpret_cast<const float4*>(ra)[c], reinterpret_cast<const float4*>(rb)[c]);
            s += (double)__fsqrt_rn(d2);
        }
    }
    // fixed-shape reduction (deterministic)
    for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
    __shared__ double red[8];
    if ((threadIdx.x & 31) == 0) red[threadIdx.x >> 5] = s;
    __syncthreads();
    if (threadIdx.x == 0) {
        double t8 = 0.0;
        for (int w = 0; w < 8; ++w) t8 += red[w];
        partial[t * gridDim.x + blockIdx.x] = t8;
    }
}

// Every block recomputes the winning trial (same fixed-order sums, so all
// agree) and gathers its slice of the winning candidates' rows.
__global__ void __launch_bounds__(512) k_landmark_pick(const double* __restrict__ partial, int nblk, int trials,
                                                      const int32_t* __restrict__ idx, int m,
                                                      const float* __restrict__ Xp, int dp,
                                                      float* __restrict__ centers) {
    __shared__ double s_tr[64];
    __shared__ int best;
    // warp w sums trial w's partials: fixed lane strides + a fixed shuffle tree (deterministic)
    const int lane = threadIdx.x & 31;
    for (int t = threadIdx.x >> 5; t < trials; t += blockDim.x >> 5) {
        double v = 0.0;
        for (int b = lane; b < nblk; b += 32) v += partial[t * nblk + b];
        for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
        if (lane == 0) s_tr[t] = v;
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        double bs = -1.0;
        int bt = 0;
        for (int t = 0; t < trials; ++t)
            if (s_tr[t] > bs) { bs = s_tr[t]; bt = t; }  // first maximum
        best = bt;
    }
    __syncthreads();
    const int32_t* w = idx + best * m;
    const int e = blockIdx.x * blockDim.x + threadIdx.x;
    if (e < m * dp) {
        const int c = e / dp, col = e - c * dp;
        centers[e] = Xp[(int64_t)w[c] * dp + col];
    }
}

// -------------------------------------------------------------- assign --
// Each thread owns one point; centers stream through shared memory. DP > 0:
// the point lives in registers (compile-time padded dimension). DP == 0:
// runtime dp, the point is re-read from L1 while 4 centers are scored at once.
template <int DP>
__global__ void __launch_bounds__(256) k_assign(const float* __restrict__ Xp, int64_t n, int dp_rt,
                                                const float* __restrict__ centers, int m, int chunk,
                                                int32_t* __restrict__ cid_out, float* __restrict__ dist_out,
                                                long long* __restrict__ sums, const double* __restrict__ fx,
                                                int32_t* __restrict__ counts) {
    extern __shared__ __align__(16) float s_c[];
    const int dp = DP > 0 ? DP : dp_rt;
    int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    bool active = i < n;
    float best = __int_as_float(0x7f800000);
    int bi = 0;
    float4 q[DP > 0 ? DP / 4 : 1];
    if constexpr (DP > 0) {
        if (active) {
#pragma unroll
            for (int c = 0; c < DP / 4; ++c) q[c] = reinterpret_cast<const float4*>(Xp + i * DP)[c];
        }
    }
    const float* xrow = Xp + (active ? i : 0) * dp;
    const bool staged = chunk > 0;  // chunk 0: high d, centers read from global memory
    const int step = staged ? chunk : m;
    for (int c0 = 0; c0 < m; c0 += step) {
        int cn = min(step, m - c0);
        const float* s_c0 = s_c;
        if (staged) {
            __syncthreads();
            for (int e = threadIdx.x; e < cn * dp / 4; e += blockDim.x)
                reinterpret_cast<float4*>(s_c)[e] = reinterpret_cast<const float4*>(centers + (int64_t)c0 * dp)[e];
            __syncthreads();
        } else {
            s_c0 = centers + (int64_t)c0 * dp;
        }
        if (!active) continue;
        if constexpr (DP > 0) {
            for (int c = 0; c < cn; ++c) {
                const float4* cc = reinterpret_cast<const float4*>(s_c0 + c * DP);
                float s = 0.f;
#pragma unroll
                for (int j = 0; j < DP / 4; ++j) s = d2_acc4(s, q[j], cc[j]);
                if (s < best) { best = s; bi = c0 + c; }
            }
        } else {
            const float4* x4 = reinterpret_cast<const float4*>(xrow);
            int c = 0;
            for (; c + 4 <= cn; c += 4) {
                float s0 = 0.f, s1 = 0.f, s2 = 0.f, s3 = 0.f;
                const float4* c4 = reinterpret_cast<const float4*>(s_c0 + c * dp);
                const int w = dp / 4;
                for (int j = 0; j < w; ++j) {
                    float4 xv = x4[j];
                    s0 = d2_acc4(s0, xv, c4[j]);
                    s1 = d2_acc4(s1, xv, c4[w + j]);
                    s2 = d2_acc4(s2, xv, c4[2 * w + j]);
                    s3 = d2_acc4(s3, xv, c4[3 * w + j]);
                }
                if (s0 < best) { best = s0; bi = c0 + c; }
                if (s1 < best) { best = s1; bi = c0 + c + 1; }
                if (s2 < best) { best = s2; bi = c0 + c + 2; }
                if (s3 < best) { best = s3; bi = c0 + c + 3; }
            }
            for (; c < cn; ++c) {
                const float4* c4 = reinterpret_cast<const float4*>(s_c0 + c * dp);
                float s = 0.f;
                for (int j = 0; j < dp / 4; ++j) s = d2_acc4(s, x4[j], c4[j]);
                if (s < best) { best = s; bi = c0 + c; }
            }
        }
    }
    if (!active) return;
    if (cid_out) cid_out[i] = bi;
    if (dist_out) dist_out[i] = __fsqrt_rn(best);
    if (counts) atomicAdd(counts + bi, 1);
    if (sums) {
        fx_accumulate(sums + (int64_t)bi * dp, xrow, dp, *fx);
    }
}

// ------------------------------------------------ center kNN graph + walk --
// The assignment only has to be approximate (reading R9: TI validity needs the
// RECORDED member-center distances to be exact, not the nearest center), so
// after the sampler the points are assigned by a greedy walk on the kNN graph
// of the centers instead of an all-centers scan (m = 3*sqrt(n) centers would
// cost n*m*d per pass). nbr[c] = the kNbr nearest centers of c (itself first).
constexpr int kNbr = 32;

// ascending bitonic sort of one key per lane across the warp
__device__ __forceinline__ key_t warp_sort32(key_t v, int lane) {
#pragma unroll
    for (int k = 2; k <= 32; k <<= 1) {
#pragma unroll
        for (int j = k >> 1; j > 0; j >>= 1) {
            const key_t o = __shfl_xor_sync(0xffffffffu, v, j);
            const bool up = (lane & k) == 0 || k == 32;
            const bool lower = (lane & j) == 0;
            v = (lower == up) ? (o < v ? o : v) : (o > v ? o : v);
        }
    }
    return v;
}

// 32-NN graph of the centers, warp per center: a batch of 32 candidate keys
// with many keys below the current 32nd (the first batches) is sorted
// (bitonic) and merged with the sorted top-32 by a bitonic half-cleaner;
// batches with few such keys insert them one by one.
__global__ void __launch_bounds__(256) k_center_knn(const float* __restrict__ centers, int m, int dp,
                                                    int32_t* __restrict__ nbr) {
    const int lane = threadIdx.x & 31;
    const int c = blockIdx.x * 8 + (threadIdx.x >> 5);
    if (c >= m) return;
    const float* rc = centers + (int64_t)c * dp;
    const int L = min(kNbr, m);
    key_t mine = (lane < 32 - L) ? kNegKey : kInfKey;  // sorted ascending across lanes
    key_t kth = kInfKey;
    // software-pipelined: the next batch's distance (its row load) is issued
    // before the current batch is merged, so the warp's 62 batches (C2) do
    // not serialise one L2 round trip each
    auto batch_key = [&](int j) -> key_t {
        return j < m ? make_key(d2_rows(rc, centers + (int64_t)j * dp, dp), j) : kInfKey;
    };
    key_t next = batch_key(lane);
    for (int base = 0; base < m; base += 32) {
        key_t key = next;
        next = batch_key(base + 32 + lane);
        unsigned cm = __ballot_sync(0xffffffffu, key_lt(key, kth));
        if (__popc(cm) <= 6) {  // few accepted keys: serial insertion
            while (cm) {
                const int src = __ffs(cm) - 1;
                const key_t kk = __shfl_sync(0xffffffffu, key, src);
                mine = warp_insert(mine, kk, lane);
                kth = __shfl_sync(0xffffffffu, mine, 31);
                cm &= ~(1u << src);
                cm &= __ballot_sync(0xffffffffu, key_lt(key, kth));
            }
            continue;
        }
        key = warp_sort32(key, lane);
        const key_t r = __shfl_sync(0xffffffffu, key, 31 - lane);  // descending
        key_t v = r < mine ? r : mine;                               // bitonic: the 32 smallest
#pragma unroll
        for (int jj = 16; jj > 0; jj >>= 1) {
            const key_t o = __shfl_xor_sync(0xffffffffu, v, jj);
            v = ((lane & jj) == 0) ? (o < v ? o : v) : (o > v ? o : v);
        }
        mine = v;
        kth = __shfl_sync(0xffffffffu, mine, 31);
    }
    if (lane >= 32 - L) nbr[(int64_t)c * kNbr + lane - (32 - L)] = key_idx(mine);
    if (lane < kNbr - L) nbr[(int64_t)c * kNbr + L + lane] = c;  // pad short lists with self
}

// Greedy walk: start at the best of the `nentry` first centers (a random
// subset: the centers are sampled points) or at the previous assignment, then
// move to the best of the current center's graph neighbours until no
// neighbour is closer. Distances are exact fp32 (direct formula), ties to the
// lower center index. Optional Lloyd accumulation and histogram.
template <int DP>
__global__ void __launch_bounds__(256) k_assign_walk(const float* __restrict__ Xp, int64_t n, int dp_rt,
                                                     const float* __restrict__ centers, int m,
                                                     const int32_t* __restrict__ nbr, int nentry,
                                                     const int32_t* __restrict__ cid_prev,
                                                     int32_t* __restrict__ cid_out, float* __restrict__ dist_out,
                                                     long long* __restrict__ sums, const double* __restrict__ fx,
                                                     int32_t* __restrict__ counts, int stride, int prev_stride,
                                                     int nwalk, int32_t* __restrict__ rank_out, int64_t base) {
    // (base: the absolute row of row 0 -- a sharded final pass covers rows
    // [base, base + n); cid_prev is valid at absolute multiples of prev_stride)
    const int dp = DP > 0 ? DP : dp_rt;
    const int64_t i = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) * stride;  // Lloyd passes subsample
    const unsigned live = __ballot_sync(0xffffffffu, i < n);  // lanes that reach the aggregated atomic
    if (i >= n) return;
    const float* xr = Xp + i * dp;
    float4 q[DP > 0 ? DP / 4 : 1];
    if constexpr (DP > 0) {
#pragma unroll
        for (int c = 0; c < DP / 4; ++c) q[c] = __ldg(reinterpret_cast<const float4*>(xr) + c);
    }
    auto dist2 = [&](int c) -> float {
        if constexpr (DP > 0) return d2_reg<DP>(q, centers + (int64_t)c * DP);
        else return d2_rows(xr, centers + (int64_t)c * dp, dp);
    };
    int best;
    float bd;
    if (cid_prev && (i + base) % prev_stride == 0) {
        best = cid_prev[i];
        bd = dist2(best);
    } else {
        best = 0;
        bd = dist2(0);
        for (int c = 1; c < nentry; ++c) {
            float v = dist2(c);
            if (v < bd) { bd = v; best = c; }
        }
    }
    for (int step = 0; step < 64; ++step) {
        const int cur = best;
        const int32_t* nb = nbr + (int64_t)cur * kNbr;
        if (nwalk == kNbr) {  // default: the whole 128-byte row in 8 vector loads, then
                              // 31 independent distances (one dependent round trip per step)
            int cs[kNbr];
#pragma unroll
            for (int j = 0; j < kNbr / 4; ++j) {
                const int4 v = __ldg(reinterpret_cast<const int4*>(nb) + j);
                cs[4 * j] = v.x; cs[4 * j + 1] = v.y; cs[4 * j + 2] = v.z; cs[4 * j + 3] = v.w;
            }
#pragma unroll
            for (int e = 1; e < kNbr; ++e) {
                const float v = dist2(cs[e]);
                if (v < bd || (v == bd && cs[e] < best)) { bd = v; best = cs[e]; }
            }
        } else {
            for (int e = 1; e < nwalk; ++e) {  // the nwalk - 1 nearest graph neighbours
                const int c = __ldg(nb + e);
                const float v = dist2(c);
                if (v < bd || (v == bd && c < best)) { bd = v; best = c; }
            }
        }
        if (best == cur) break;
    }
    if (cid_out) cid_out[i] = best;
    if (dist_out) dist_out[i] = __fsqrt_rn(bd);
    if (counts) {  // rank_out: the member's slot in its cluster (k_scatter_keys needs no atomics)
        // warp-aggregated: lanes with the same cluster (neighbouring input rows
        // often share one) take one atomic; slots are sorted away later, so the
        // order within a group does not matter
        const int lane = threadIdx.x & 31;
        const unsigned grp = __match_any_sync(live, best);
        const int leader = __ffs(grp) - 1;
        int base = 0;
        if (lane == leader) base = atomicAdd(counts + best, __popc(grp));
        base = __shfl_sync(grp, base, leader);
        if (rank_out) rank_out[i] = base + __popc(grp & ((1u << lane) - 1u));
    }
    if (sums) {
        fx_accumulate(sums + (int64_t)best * dp, xr, dp, *fx);
    }
}

// ------------------------------------------------------------ D^2 seeding --
// sum of squared distances, deterministic: per-block partials + ordered final sum
__global__ void k_sum_sq(const float* __restrict__ dist, int64_t n, double* __restrict__ partial) {
    double s = 0.0;
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
        const double v = dist[i];
        s += v * v;
    }
    __shared__ double red[256];
    red[threadIdx.x] = s;
    __syncthreads();
    for (int w = blockDim.x / 2; w > 0; w >>= 1) {
        if (threadIdx.x < w) red[threadIdx.x] += red[threadIdx.x + w];
        __syncthreads();
    }
    if (threadIdx.x == 0) partial[blockIdx.x] = red[0];
}

__global__ void k_sum_final(const double* __restrict__ partial, int nb, double* __restrict__ out) {
    __shared__ double red[256];
    double v = 0.0;
    for (int b = threadIdx.x; b < nb; b += blockDim.x) v += partial[b];
    red[threadIdx.x] = v;
    __syncthreads();
    for (int w = blockDim.x / 2; w > 0; w >>= 1) {
        if (threadIdx.x < w) red[threadIdx.x] += red[threadIdx.x + w];
        __syncthreads();
    }
    if (threadIdx.x == 0) *out = red[0];
}

// point i becomes a center with probability min(1, m1 * d2_i / S); the picks
// are compacted in point order (count -> scan -> write), so the sampled set
// and its slot order are deterministic.
constexpr int kSampleBlocks = 1024;

__device__ __forceinline__ bool d2_pick(const float* __restrict__ dist, int64_t i, double tot, int m1, uint64_t seed) {
    const double v = dist[i];
    const double p = (double)m1 * v * v / tot;
    const double u = (double)mix32(seed * 0x2545f4914f6cdd1dull + (uint64_t)i) * (1.0 / 4294967296.0);
    return u < p;
}

__global__ void __launch_bounds__(256) k_d2_count(const float* __restrict__ dist, int64_t n, const double* __restrict__ S,
                                                  int m1, uint64_t seed, int32_t* __restrict__ bcount) {
    const double tot = *S;
    const int64_t per = (n + gridDim.x - 1) / gridDim.x;
    const int64_t lo = blockIdx.x * per, hi = min(n, lo + per);
    int c = 0;
    if (tot > 0.0)
        for (int64_t i = lo + threadIdx.x; i < hi; i += blockDim.x) c += d2_pick(dist, i, tot, m1, seed) ? 1 : 0;
    for (int o = 16; o > 0; o >>= 1) c += __shfl_xor_sync(0xffffffffu, c, o);
    __shared__ int red[8];
    if ((threadIdx.x & 31) == 0) red[threadIdx.x >> 5] = c;
    __syncthreads();
    if (threadIdx.x == 0) {
        int t = 0;
        for (int w = 0; w < 8; ++w) t += red[w];
        bcount[blockIdx.x] = t;
    }
}

__global__ void __launch_bounds__(256) k_d2_write(const float* __restrict__ Xp, int64_t n, int dp,
                                                  const float* __restrict__ dist, const double* __restrict__ S, int m1,
                                                  uint64_t seed, const int32_t* __restrict__ boff,
                                                  float* __restrict__ centers) {
    const double tot = *S;
    if (!(tot > 0.0)) return;
    const int64_t per = (n + gridDim.x - 1) / gridDim.x;
    const int64_t lo = blockIdx.x * per, hi = min(n, lo + per);
    __shared__ int wc[8];
    int run = boff[blockIdx.x];
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    for (int64_t base = lo; base < hi; base += blockDim.x) {
        const int64_t i = base + threadIdx.x;
        const bool pick = i < hi && d2_pick(dist, i, tot, m1, seed);
        const unsigned bm = __ballot_sync(0xffffffffu, pick);
        if (lane == 0) wc[w] = __popc(bm);
        __syncthreads();
        int off = run;
        for (int ww = 0; ww < w; ++ww) off += wc[ww];
        if (pick) {
            const int slot = off + __popc(bm & ((1u << lane) - 1u));
            if (slot < m1) {
                const float4* src = reinterpret_cast<const float4*>(Xp + i * dp);
                float4* dst = reinterpret_cast<float4*>(centers + (int64_t)slot * dp);
                for (int c = 0; c < dp / 4; ++c) dst[c] = src[c];
            }
        }
        for (int ww = 0; ww < 8; ++ww) run += wc[ww];
        __syncthreads();
    }
}

// slots the sampling left empty get random points
__global__ void k_d2_fill(const float* __restrict__ Xp, int64_t n, int dp, int m1, uint64_t seed,
                          float* __restrict__ centers, const int32_t* __restrict__ total) {
    const int start = min(*total, m1);
    for (int j = start + blockIdx.x * blockDim.x + threadIdx.x; j < m1; j += gridDim.x * blockDim.x) {
        const uint32_t i = perm_index((uint32_t)j, (uint32_t)n, seed ^ 0xd2d2d2d2ull);
        const float4* src = reinterpret_cast<const float4*>(Xp + (int64_t)i * dp);
        float4* dst = reinterpret_cast<float4*>(centers + (int64_t)j * dp);
        for (int c = 0; c < dp / 4; ++c) dst[c] = src[c];
    }
}

// Lloyd update from the fixed-point sums (deterministic: integer adds commute)
// one thread per center; the sums and counts are zeroed after use, ready for
// the next pass (no memsets between passes)
__global__ void k_lloyd_update(float* __restrict__ centers, long long* __restrict__ sums,
                               const double* __restrict__ fx, int32_t* __restrict__ counts, int m, int dp) {
    const double inv = 1.0 / *fx;
    for (int c = blockIdx.x * blockDim.x + threadIdx.x; c < m; c += gridDim.x * blockDim.x) {
        const int cnt = counts[c];
        for (int j = 0; j < dp; ++j) {
            const int64_t e = (int64_t)c * dp + j;
            if (cnt > 0) centers[e] = (float)((double)sums[e] * inv / (double)cnt);
            sums[e] = 0;
        }
        counts[c] = 0;
    }
}

// fixed-point scale for the Lloyd sums: 2^s with max|x| * n * 2^s < 2^61
// max |x| over the padded rows (total = n * dp, a multiple of 4): float4
// loads, one shared-memory and one global atomic per CTA
__global__ void __launch_bounds__(256) k_absmax(const float* __restrict__ Xp, int64_t total,
                                                unsigned int* __restrict__ out) {
    __shared__ unsigned s_mx;
    if (threadIdx.x == 0) s_mx = 0u;
    __syncthreads();
    float mx = 0.f;
    const float4* X4 = reinterpret_cast<const float4*>(Xp);
    for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < total / 4; e += (int64_t)gridDim.x * blockDim.x) {
        const float4 v = __ldg(X4 + e);
        mx = fmaxf(mx, fmaxf(fmaxf(fabsf(v.x), fabsf(v.y)), fmaxf(fabsf(v.z), fabsf(v.w))));
    }
    for (int o = 16; o > 0; o >>= 1) mx = fmaxf(mx, __shfl_xor_sync(0xffffffffu, mx, o));
    if ((threadIdx.x & 31) == 0) atomicMax(&s_mx, __float_as_uint(mx));
    __syncthreads();
    if (threadIdx.x == 0) atomicMax(out, s_mx);
}

__global__ void k_fx_scale(const unsigned int* __restrict__ amax, int64_t n, double* __restrict__ fx) {
    const double mx = fmax((double)__uint_as_float(*amax), 1e-30);
    const double e = floor(61.0 - log2(mx * (double)n));
    *fx = exp2(fmin(e, 1000.0));
}

// --------------------------------------------------------------- CSR -----
// Single-CTA exclusive scan of cluster counts -> off[0..m]; zeroes cursor.
__global__ void __launch_bounds__(1024) k_offsets(const int32_t* __restrict__ counts, int m, int32_t* __restrict__ off,
                                                  int32_t* __restrict__ cursor) {
    __shared__ int32_t s_sum[1024];
    __shared__ int32_t s_carry;
    if (threadIdx.x == 0) s_carry = 0;
    __syncthreads();
    for (int base = 0; base < m; base += 1024) {
        int i = base + threadIdx.x;
        int v = (i < m) ? counts[i] : 0;
        s_sum[threadIdx.x] = v;
        __syncthreads();
        for (int w = 1; w < 1024; w <<= 1) {  // Hillis-Steele inclusive scan
            int t = (threadIdx.x >= w) ? s_sum[threadIdx.x - w] : 0;
            __syncthreads();
            s_sum[threadIdx.x] += t;
            __syncthreads();
        }
        if (i < m) {
            off[i] = s_carry + s_sum[threadIdx.x] - v;
            cursor[i] = 0;
        }
        __syncthreads();
        if (threadIdx.x == 1023) s_carry += s_sum[1023];
        __syncthreads();
    }
    if (threadIdx.x == 0) off[m] = s_carry;
}

// key: (~dist_bits) << 32 | index -> ascending key = descending distance, ascending index
// rank (optional): slots already taken by the assignment's histogram atomics
__global__ void k_scatter_keys(const int32_t* __restrict__ cid, const float* __restrict__ dist, int64_t n,
                               const int32_t* __restrict__ off, int32_t* __restrict__ cursor,
                               const int32_t* __restrict__ rank, u64* __restrict__ keys) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
        int c = cid[i];
        int pos = off[c] + (rank ? rank[i] : atomicAdd(cursor + c, 1));
        keys[pos] = (u64(~__float_as_uint(dist[i])) << 32) | u64(uint32_t(i));
    }
}

__device__ __forceinline__ float key_member_dist(u64 key) { return __uint_as_float(~uint32_t(key >> 32)); }

// Ascending bitonic network in the "flip + half-cleaner" form: every
// compare-exchange puts the minimum at the lower index, so virtual +inf
// padding past the segment end never moves (no padding writes needed).
__device__ __forceinline__ void cmpx(u64* s, int i, int p) {
    u64 a = s[i], b = s[p];
    if (b < a) { s[i] = b; s[p] = a; }
}

constexpr int kSmallSeg = 4096;  // smem chunk of k_segsort_big
constexpr int kTinySeg = 256;    // register sort in k_segsort_small (one warp, 8 keys per lane)

// Segments of up to 32*R keys: one warp, R keys per lane in registers
// (element e = r*32 + lane), the same ascending bitonic network with
// partners e ^ j: shuffles for j < 32, in-thread exchanges for j >= 32.
// No shared memory, no barriers (ncu, C2: the 128-thread smem network
// issued 12.4M warp instructions for 1978 clusters of ~220 keys).
template <int R>
__device__ __forceinline__ void warp_segsort(u64* __restrict__ g, int size, float* __restrict__ radius_out) {
    const int lane = threadIdx.x & 31;
    u64 v[R];
#pragma unroll
    for (int r = 0; r < R; ++r) v[r] = (r * 32 + lane < size) ? g[r * 32 + lane] : ~0ull;
#pragma unroll
    for (int k = 2; k <= 32 * R; k <<= 1) {
#pragma unroll
        for (int j = k >> 1; j > 0; j >>= 1) {
            if (j >= 32) {  // k >= 64: the direction depends on the register index only
#pragma unroll
                for (int r = 0; r < R; ++r) {
                    if (r & (j >> 5)) continue;
                    const int p = r | (j >> 5);
                    const bool asc = ((r * 32) & k) == 0;
                    const u64 a = v[r], b = v[p];
                    const bool sw = asc ? (b < a) : (a < b);
                    v[r] = sw ? b : a;
                    v[p] = sw ? a : b;
                }
            } else {
#pragma unroll
                for (int r = 0; r < R; ++r) {
                    const u64 o = __shfl_xor_sync(0xffffffffu, v[r], j);
                    const bool asc = ((r * 32 + lane) & k) == 0;
                    const bool lower = (lane & j) == 0;
                    v[r] = (lower == asc) ? (o < v[r] ? o : v[r]) : (o > v[r] ? o : v[r]);
                }
            }
        }
    }
#pragma unroll
    for (int r = 0; r < R; ++r)
        if (r * 32 + lane < size) g[r * 32 + lane] = v[r];
    if (lane == 0) *radius_out = key_member_dist(v[0]);
}

// one 256-thread CTA per cluster of at most kMidSeg members: up to kTinySeg
// members warp 0 sorts in registers (the other warps leave), larger clusters
// run the bitonic network in 8 KB of shared memory. (Measured and rejected:
// 8 clusters per CTA, one warp each, with the 257-1024-member ones in a second
// launch -- C2 25.5 -> 38 us; register sorts up to 512 members -- 62 us.)
constexpr int kMidSeg = 1024;
__global__ void __launch_bounds__(256) k_segsort_small(u64* __restrict__ keys, const int32_t* __restrict__ off,
                                                       float* __restrict__ radius) {
    __shared__ u64 s[kMidSeg];
    const int c = blockIdx.x;
    const int lo = off[c], size = off[c + 1] - lo;
    if (size > kMidSeg) return;
    if (size <= 1) {
        if (threadIdx.x == 0) radius[c] = size ? key_member_dist(keys[lo]) : 0.f;
        return;
    }
    if (size <= kTinySeg) {  // uniform per CTA
        if (threadIdx.x >= 32) return;
        if (size <= 32) warp_segsort<1>(keys + lo, size, radius + c);
        else if (size <= 64) warp_segsort<2>(keys + lo, size, radius + c);
        else if (size <= 128) warp_segsort<4>(keys + lo, size, radius + c);
        else warp_segsort<8>(keys + lo, size, radius + c);
        return;
    }
    int S = 2;
    while (S < size) S <<= 1;
    for (int i = threadIdx.x; i < S; i += blockDim.x) s[i] = (i < size) ? keys[lo + i] : ~0ull;
    __syncthreads();
    for (int k = 2, lk = 1; k <= S; k <<= 1, ++lk) {
        for (int t = threadIdx.x; t < S / 2; t += blockDim.x) {  // flip
            const int blk = t >> (lk - 1), r = t & (k / 2 - 1);
            const int i = (blk << lk) + r, p = (blk << lk) + k - 1 - r;
            cmpx(s, i, p);
        }
        __syncthreads();
        for (int j = k / 4, lj = lk - 2; j > 0; j >>= 1, --lj) {  // half-cleaners
            for (int t = threadIdx.x; t < S / 2; t += blockDim.x) {
                const int i = ((t >> lj) << (lj + 1)) + (t & (j - 1));
                cmpx(s, i, i + j);
            }
            __syncthreads();
        }
    }
    for (int i = threadIdx.x; i < size; i += blockDim.x) keys[lo + i] = s[i];
    if (threadIdx.x == 0) radius[c] = key_member_dist(s[0]);
}

// Clusters larger than kMidSeg: one CTA per cluster (up to kSmallSeg the
// whole segment sorts in smem in phase A); stages whose partner
// distance is < kSmallSeg run in shared memory chunk by chunk, the others
// directly on global memory (virtual +inf padding beyond the segment).
__global__ void __launch_bounds__(1024) k_segsort_big(u64* __restrict__ keys, const int32_t* __restrict__ off,
                                                      float* __restrict__ radius) {
    __shared__ u64 s[kSmallSeg];
    int c = blockIdx.x;
    int lo = off[c], size = off[c + 1] - lo;
    if (size <= kMidSeg) return;
    u64* g = keys + lo;
    int S = 2;
    while (S < size) S <<= 1;
    auto gx = [&](int i, int p) {
        if (p >= size) return;
        u64 a = g[i], b = g[p];
        if (b < a) { g[i] = b; g[p] = a; }
    };
    // phase A: fully sort every aligned chunk of CL = min(kSmallSeg, S) keys in smem
    const int CL = S < kSmallSeg ? S : kSmallSeg;
    for (int base = 0; base < size; base += CL) {
        for (int i = threadIdx.x; i < CL; i += blockDim.x) s[i] = (base + i < size) ? g[base + i] : ~0ull;
        __syncthreads();
        for (int k = 2, lk = 1; k <= CL; k <<= 1, ++lk) {
            for (int t = threadIdx.x; t < CL / 2; t += blockDim.x) {
                const int blk = t >> (lk - 1), r = t & (k / 2 - 1);
                cmpx(s, (blk << lk) + r, (blk << lk) + k - 1 - r);
            }
            __syncthreads();
            for (int j = k / 4, lj = lk - 2; j > 0; j >>= 1, --lj) {
                for (int t = threadIdx.x; t < CL / 2; t += blockDim.x) {
                    const int i = ((t >> lj) << (lj + 1)) + (t & (j - 1));
                    cmpx(s, i, i + j);
                }
                __syncthreads();
            }
        }
        for (int i = threadIdx.x; i < CL && base + i < size; i += blockDim.x) g[base + i] = s[i];
        __syncthreads();
    }
    // phase B: merges of size > kSmallSeg
    for (int k = 2 * kSmallSeg, lk = __ffs(2 * kSmallSeg) - 1; k <= S; k <<= 1, ++lk) {
        for (int t = threadIdx.x; t < S / 2; t += blockDim.x) {
            const int blk = t >> (lk - 1), r = t & (k / 2 - 1);  // powers of two: shifts, not divisions
            const int i = (blk << lk) + r, p = (blk << lk) + k - 1 - r;
            if (i < size) gx(i, p);
        }
        __syncthreads();
        for (int j = k / 4, lj = lk - 2; j >= kSmallSeg; j >>= 1, --lj) {
            for (int t = threadIdx.x; t < S / 2; t += blockDim.x) {
                const int i = ((t >> lj) << (lj + 1)) + (t & (j - 1));
                if (i < size) gx(i, i + j);
            }
            __syncthreads();
        }
        // remaining half-cleaners (j < kSmallSeg) stay inside aligned chunks
        for (int base = 0; base < size; base += kSmallSeg) {
            for (int i = threadIdx.x; i < kSmallSeg; i += blockDim.x) s[i] = (base + i < size) ? g[base + i] : ~0ull;
            __syncthreads();
            for (int jj = kSmallSeg / 2, ljj = __ffs(kSmallSeg / 2) - 1; jj > 0; jj >>= 1, --ljj) {
                for (int t = threadIdx.x; t < kSmallSeg / 2; t += blockDim.x) {
                    const int i = ((t >> ljj) << (ljj + 1)) + (t & (jj - 1));
                    cmpx(s, i, i + jj);
                }
                __syncthreads();
            }
            for (int i = threadIdx.x; i < kSmallSeg && base + i < size; i += blockDim.x) g[base + i] = s[i];
            __syncthreads();
        }
    }
    if (threadIdx.x == 0) radius[c] = key_member_dist(g[0]);
}

// per-cluster summary read by level-1 and the scan with one 16-byte load:
// {lo, hi, radius, smallest member distance} (the last member: R11 order)
__global__ void k_side_info(const int32_t* __restrict__ off, const float* __restrict__ radius,
                            const float* __restrict__ dist, int m, int4* __restrict__ tinfo) {
    const int c = blockIdx.x * blockDim.x + threadIdx.x;
    if (c >= m) return;
    const int lo = off[c], hi = off[c + 1];
    const float dmin = hi > lo ? dist[hi - 1] : __int_as_float(0x7f800000);
    tinfo[c] = make_int4(lo, hi, __float_as_int(radius[c]), __float_as_int(dmin));
}

// rows_out[p] = Xp[idx(p)], dist_out[p], orig_out[p]; one thread per float4
__global__ void k_gather_side(const u64* __restrict__ keys, const float* __restrict__ Xp, int64_t n, int dp,
                              float* __restrict__ rows_out, float* __restrict__ dist_out, int32_t* __restrict__ orig_out) {
    const int w = dp / 4;
    int64_t total = n * w;
    for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < total; e += (int64_t)gridDim.x * blockDim.x) {
        int64_t p = e / w;
        int c = int(e - p * w);
        u64 key = keys[p];
        uint32_t idx = uint32_t(key & 0xffffffffu);
        reinterpret_cast<float4*>(rows_out)[e] = reinterpret_cast<const float4*>(Xp)[(int64_t)idx * w + c];
        if (c == 0) {
            dist_out[p] = key_member_dist(key);
            orig_out[p] = (int32_t)idx;
        }
    }
}

// ------------------------------------------------------------ launcher --
// centers per shared-memory chunk of the SIMT assignment; 0 = high d (a row
// above 48 KB): the centers are read from global memory, no staging
static int assign_chunk(int dp, int m, size_t* smem) {
    int chunk = int((48 * 1024) / (dp * sizeof(float)));
    if (chunk > m) chunk = m;
    if (chunk < 1) {
        *smem = 0;
        return 0;
    }
    *smem = size_t(chunk) * dp * sizeof(float);
    return chunk;
}

static void launch_assign(Ctx& cx, const float* Xp, int64_t n, int dp, const float* centers, int m,
                          int32_t* cid, float* dist, long long* sums, const double* fx, int32_t* counts) {
    size_t smem;
    int chunk = assign_chunk(dp, m, &smem);
    dim3 grid((unsigned)((n + 255) / 256));
    switch (dp) {
#define SKNN_ASSIGN_CASE(D) \
    case D: k_assign<D><<<grid, 256, smem, cx.stream>>>(Xp, n, dp, centers, m, chunk, cid, dist, sums, fx, counts); break;
        SKNN_ASSIGN_CASE(4) SKNN_ASSIGN_CASE(8) SKNN_ASSIGN_CASE(12) SKNN_ASSIGN_CASE(16)
        SKNN_ASSIGN_CASE(20) SKNN_ASSIGN_CASE(24) SKNN_ASSIGN_CASE(28) SKNN_ASSIGN_CASE(32)
#undef SKNN_ASSIGN_CASE
        default: k_assign<0><<<grid, 256, smem, cx.stream>>>(Xp, n, dp, centers, m, chunk, cid, dist, sums, fx, counts); break;
    }
    cx.launched();
}

// Build one clustered side (Step 1). X is a device pointer [n x d].
__global__ void k_histogram(const int32_t* __restrict__ cid, int64_t n, int32_t* __restrict__ counts) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        atomicAdd(counts + cid[i], 1);
}

sknn_status build_side(Ctx& cx, const float* X, int64_t n, int d, int m, int trials, int lloyd, uint64_t seed,
                       Side& out, const BuildShard* shard) {
    const int mode = shard ? shard->mode : 0;
    const bool from_asg = mode == 2;  // the clustering is given: no sampler, no Lloyd, no assignment
    const int dp = (d + 3) & ~3;
    out.n = n; out.d = d; out.dp = dp; out.m = m;
    cudaStream_t s = cx.stream;
    // owned outputs
    SKNN_TRY(cx.alloc_persistent((void**)&out.rows, sizeof(float) * n * dp));
    SKNN_TRY(cx.alloc_persistent((void**)&out.dist, sizeof(float) * n));
    SKNN_TRY(cx.alloc_persistent((void**)&out.orig, sizeof(int32_t) * n));
    SKNN_TRY(cx.alloc_persistent((void**)&out.off, sizeof(int32_t) * (m + 1)));
    SKNN_TRY(cx.alloc_persistent((void**)&out.centers, sizeof(float) * m * dp));
    SKNN_TRY(cx.alloc_persistent((void**)&out.radius, sizeof(float) * m));
    SKNN_TRY(cx.alloc_persistent((void**)&out.tinfo, sizeof(int4) * m));
    out.owned = true;

    // padded copy of X (skipped when X already has 16-byte rows)
    const float* Xp = X;
    if (dp != d || (reinterpret_cast<uintptr_t>(X) & 15u)) {
        float* tmp;
        SKNN_TRY(cx.alloc_scratch((void**)&tmp, sizeof(float) * n * dp));
        int64_t tot = n * dp;
        int blocks = (int)std::min<int64_t>((tot + 255) / 256, 148 * 16);
        k_pad_rows<<<blocks, 256, 0, s>>>(X, n, d, dp, tmp);
        cx.launched();
        Xp = tmp;
    }
    // D^2 seeding split (reading R9): m0 landmarks from the paper's sampler
    // (P:L321), the other m - m0 drawn with probability ~ squared distance to
    // the nearest landmark (one k-means|| round), so small or far groups of
    // points get a center instead of inflating a far cluster's radius.
    const char* sd = getenv("SKNN_SEEDING");
    // (measured: helps dp >= 16 -- C3 202 -> 137 candidate clusters -- and is
    // neutral for the low-dimensional C1/C2, where it only costs a pass)
    const bool d2seed = !(sd && strcmp(sd, "paper") == 0) && m >= 64 && (dp >= 16 || (sd && strcmp(sd, "d2") == 0));
    const int m0 = d2seed ? (m + 1) / 2 : m;
    // landmark sampler
    int32_t* lidx;
    SKNN_TRY(cx.alloc_scratch((void**)&lidx, sizeof(int32_t) * trials * m0));
    if (!from_asg) {
        k_landmark_draw<<<dim3((m0 + 255) / 256, trials), 256, 0, s>>>(n, m0, trials, seed, lidx);
        cx.launched();
    }
    const int nb = (m0 + kLmTile - 1) / kLmTile;
    const int ntile = nb * (nb + 1) / 2;
    double* partial;
    SKNN_TRY(cx.alloc_scratch((void**)&partial, sizeof(double) * trials * ntile));
    size_t lsm = dp <= 128 ? sizeof(float) * 2 * kLmTile * dp : 0;
    if (lsm > 48 * 1024)
        SKNN_CUDA(cudaFuncSetAttribute(k_landmark_sums, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)lsm));
    // (measured and rejected: one CTA per (trial, 1/16 or 1/64 of the rows)
    // with the whole trial staged in shared memory -- C2 61 / 52 us vs 30 us)
    if (!from_asg) {
        k_landmark_sums<<<dim3(ntile, trials), 256, lsm, s>>>(Xp, dp, m0, lidx, nb, partial);
        cx.launched();
        k_landmark_pick<<<(m0 * dp + 511) / 512, 512, 0, s>>>(partial, ntile, trials, lidx, m0, Xp, dp, out.centers);
        cx.launched();
    }

    int32_t* cid;
    float* pdist;
    int32_t* counts;
    int32_t* cursor;
    SKNN_TRY(cx.alloc_scratch((void**)&cid, sizeof(int32_t) * n));
    SKNN_TRY(cx.alloc_scratch((void**)&pdist, sizeof(float) * n));
    SKNN_TRY(cx.alloc_scratch((void**)&counts, sizeof(int32_t) * m));
    SKNN_TRY(cx.alloc_scratch((void**)&cursor, sizeof(int32_t) * m));
    // assignment (approximate is enough, R9): tensor-core screen over all
    // centers for dp >= 16 (k_assign_tc), greedy walk on the center kNN graph
    // for low dp, exact all-centers SIMT scan otherwise. SKNN_ASSIGN=
    // tc|walk|full overrides (ablation).
    const char* am = getenv("SKNN_ASSIGN");
    const bool force_full = am && strcmp(am, "full") == 0;
    const bool force_walk = am && strcmp(am, "walk") == 0;
    const bool force_tc = am && strcmp(am, "tc") == 0;
    const bool use_tc = !force_full && !force_walk && assign_tc_supported(dp) && (force_tc || dp >= 16);
    const bool walk = !use_tc && !force_full && m > kNbr;
    int32_t* nbr = nullptr;
    if (walk) SKNN_TRY(cx.alloc_scratch((void**)&nbr, sizeof(int32_t) * (size_t)m * kNbr));
    const char* ne = getenv("SKNN_WALK_ENTRIES");
    const int nentry = std::min(m0, ne ? std::max(1, atoi(ne)) : 64);
    // fixed-point scale of the Lloyd sums (deterministic centers, hence a
    // deterministic clustering: query-sharded ranks agree on cluster ids)
    double* fx;
    unsigned int* amax;
    SKNN_TRY(cx.alloc_scratch((void**)&fx, sizeof(double) + sizeof(unsigned int)));
    amax = reinterpret_cast<unsigned int*>(fx + 1);
    if (lloyd > 0 && !from_asg) {
        SKNN_CUDA(cudaMemsetAsync(amax, 0, sizeof(unsigned int), s));
        k_absmax<<<(int)std::min<int64_t>((n * dp / 4 + 255) / 256, 148 * 2), 256, 0, s>>>(Xp, n * dp, amax);
        k_fx_scale<<<1, 1, 0, s>>>(amax, n, fx);
        cx.launched();
        cx.launched();
    }
    const float* Xp_all = Xp;
    int graph_m = -1;
    int32_t* rank_o = nullptr;  // set for the final walk pass only
    // rows the next assignment pass covers: all, or (mode 1, final pass) [alo, alo + an)
    int64_t alo = 0, an = n;
    auto assign = [&](const int32_t* prev, int32_t* cid_o, float* dist_o, long long* sums_o, int mc, int stride,
                      int prev_stride) -> sknn_status {
        const float* Xp = Xp_all + alo * dp;  // (alo is a multiple of every stride: 8)
        const int64_t n = an;
        if (prev) prev += alo;
        if (cid_o) cid_o += alo;
        if (dist_o) dist_o += alo;
        if (use_tc) return run_assign_tc(cx, Xp, n, dp, out.centers, mc, cid_o, dist_o, sums_o, fx, counts, stride);
        if (!walk || mc <= kNbr) {
            launch_assign(cx, Xp, n, dp, out.centers, mc, cid_o, dist_o, sums_o, fx, counts);
            return SKNN_OK;
        }
        // the walk may use a slightly stale graph (the assignment only has to be
        // approximate): build it for the first pass and after seeding only
        if (graph_m != mc) {
            // (measured and rejected: centers staged in shared memory, two-pass
            // bound + compaction, 16 warps per CTA -- C2 29.5 vs 30.5 us)
            // (measured and rejected: each center's candidates split over 4 warps
            // merged bitonically -- C2 30 -> 41 us)
            k_center_knn<<<(mc + 7) / 8, 256, 0, s>>>(out.centers, mc, dp, nbr);
            cx.launched();
            graph_m = mc;
        }
        dim3 grid((unsigned)(((n + stride - 1) / stride + 255) / 256));
        // graph neighbours tried per walk step (ablation; measured on C2: 24 -> +3%,
        // 16 -> +17%, 8 -> +88% join time, the worse clustering costs the scan more)
        const char* wn = getenv("SKNN_WALK_NBR");
        const int nwalk = wn ? std::max(2, std::min(kNbr, atoi(wn))) : kNbr;
        switch (dp) {
#define SKNN_WALK_CASE(D)                                                                                      \
    case D:                                                                                                    \
        k_assign_walk<D><<<grid, 256, 0, s>>>(Xp, n, dp, out.centers, mc, nbr, nentry, prev, cid_o, dist_o, sums_o, \
                                              fx, counts, stride, prev_stride, nwalk, rank_o, alo);                 \
        break;
            SKNN_WALK_CASE(4) SKNN_WALK_CASE(8) SKNN_WALK_CASE(12) SKNN_WALK_CASE(16)
            SKNN_WALK_CASE(20) SKNN_WALK_CASE(24) SKNN_WALK_CASE(28) SKNN_WALK_CASE(32)
#undef SKNN_WALK_CASE
            default:
                k_assign_walk<0><<<grid, 256, 0, s>>>(Xp, n, dp, out.centers, mc, nbr, nentry, prev, cid_o, dist_o,
                                                      sums_o, fx, counts, stride, prev_stride, nwalk, rank_o, alo);
                break;
        }
        cx.launched();
        return SKNN_OK;
    };
    const int32_t* prev = nullptr;
    // the D^2 draw only needs the squared distances of a sample: the seeding
    // pass assigns every sstride-th point (others keep distance 0 = never drawn;
    // C5 build 21.2 -> 17.1 ms for both sides, C3 join 3.94 -> 3.65 ms)
    // (dp <= 32 only: at d = 128 (C4) the sampled seeding let a few clusters grow
    // large and the warp-per-query scan's tail explode -- measured 25 -> 824 ms)
    // (study knob SKNN_SUBSAMPLE_HIGHD=1: strided seeding / Lloyd passes also above dp 32)
    static const bool sub_highd = getenv("SKNN_SUBSAMPLE_HIGHD") != nullptr;
    const bool subsample = dp <= 32 || sub_highd;
    const int sstride = subsample ? (int)std::max<int64_t>(1, std::min<int64_t>(8, n / (64LL * std::max(1, m0)))) : 1;
    int seed_stride = 1;
    if (m0 < m && !from_asg) {
        SKNN_CUDA(cudaMemsetAsync(counts, 0, sizeof(int32_t) * m, s));
        if (sstride > 1) SKNN_CUDA(cudaMemsetAsync(pdist, 0, sizeof(float) * n, s));
        SKNN_TRY(assign(nullptr, cid, pdist, nullptr, m0, sstride, 1));
        prev = cid;
        seed_stride = sstride;
        double* ssum;
        int32_t* bcnt;
        int32_t* boff;
        const int rb = (int)std::min<int64_t>((n + 255) / 256, 148 * 8);
        SKNN_TRY(cx.alloc_scratch((void**)&ssum, sizeof(double) * (rb + 1)));
        SKNN_TRY(cx.alloc_scratch((void**)&bcnt, sizeof(int32_t) * (3 * kSampleBlocks + 8)));
        boff = bcnt + kSampleBlocks;                   // kSampleBlocks + 1 entries
        int32_t* dummy = bcnt + 2 * kSampleBlocks + 1;  // cursor scratch of k_offsets
        k_sum_sq<<<rb, 256, 0, s>>>(pdist, n, ssum + 1);
        cx.launched();
        k_sum_final<<<1, 256, 0, s>>>(ssum + 1, rb, ssum);
        cx.launched();
        k_d2_count<<<kSampleBlocks, 256, 0, s>>>(pdist, n, ssum, m - m0, seed, bcnt);
        cx.launched();
        k_offsets<<<1, 1024, 0, s>>>(bcnt, kSampleBlocks, boff, dummy);
        cx.launched();
        k_d2_write<<<kSampleBlocks, 256, 0, s>>>(Xp, n, dp, pdist, ssum, m - m0, seed, boff,
                                                 out.centers + (int64_t)m0 * dp);
        cx.launched();
        k_d2_fill<<<std::max(1, (m - m0 + 255) / 256), 256, 0, s>>>(Xp, n, dp, m - m0, seed, out.centers + (int64_t)m0 * dp,
                                                                   boff + kSampleBlocks);
        cx.launched();
    }
    // Lloyd iterations (R9) on a strided subsample (~64+ points per cluster):
    // the centers only have to be good, not exact (mini-batch k-means)
    // (measured: neutral-to-better for dp <= 32; at d = 128 (C4) the subsampled
    // centers let a few clusters grow large and the scan's tail suffers)
    const int lstride = subsample ? (int)std::max<int64_t>(1, std::min<int64_t>(8, n / (64LL * m))) : 1;
    int prev_stride = seed_stride;  // cid entries valid at multiples of it
    if (lloyd > 0 && !from_asg) {
        long long* sums;
        SKNN_TRY(cx.alloc_scratch((void**)&sums, sizeof(long long) * m * dp));
        SKNN_CUDA(cudaMemsetAsync(sums, 0, sizeof(long long) * m * dp, s));
        SKNN_CUDA(cudaMemsetAsync(counts, 0, sizeof(int32_t) * m, s));
        for (int it = 0; it < lloyd; ++it) {  // k_lloyd_update re-zeroes sums and counts
            SKNN_TRY(assign(prev, cid, nullptr, sums, m, lstride, prev ? prev_stride : 1));
            prev = cid;
            prev_stride = lstride;
            k_lloyd_update<<<(m + 127) / 128, 128, 0, s>>>(out.centers, sums, fx, counts, m, dp);
            cx.launched();
        }
    }
    // final assignment with exact member distances + histogram
    if (lloyd <= 0 || from_asg) SKNN_CUDA(cudaMemsetAsync(counts, 0, sizeof(int32_t) * m, s));
    if (from_asg) {  // mode 2: the gathered clustering
        SKNN_CUDA(cudaMemcpyAsync(out.centers, shard->centers_in, sizeof(float) * m * dp, cudaMemcpyDeviceToDevice, s));
        SKNN_CUDA(cudaMemcpyAsync(cid, shard->cid_in, sizeof(int32_t) * n, cudaMemcpyDeviceToDevice, s));
        SKNN_CUDA(cudaMemcpyAsync(pdist, shard->dist_in, sizeof(float) * n, cudaMemcpyDeviceToDevice, s));
        k_histogram<<<(int)std::min<int64_t>((n + 255) / 256, 148 * 8), 256, 0, s>>>(cid, n, counts);
        cx.launched();
    } else if (mode == 1) {  // this rank's rows of the final assignment, then stop
        alo = shard->lo;
        an = shard->hi - shard->lo;
        if (an > 0) SKNN_TRY(assign(prev, cid, pdist, nullptr, m, 1, prev_stride));
        SKNN_CUDA(cudaMemcpyAsync(shard->centers_out, out.centers, sizeof(float) * m * dp, cudaMemcpyDeviceToDevice, s));
        if (an > 0) {
            SKNN_CUDA(cudaMemcpyAsync(shard->cid_out + alo, cid + alo, sizeof(int32_t) * an, cudaMemcpyDeviceToDevice, s));
            SKNN_CUDA(cudaMemcpyAsync(shard->dist_out + alo, pdist + alo, sizeof(float) * an, cudaMemcpyDeviceToDevice, s));
        }
        return cx.check_launch("build_side (assignment shard)");
    } else {
        if (walk) SKNN_TRY(cx.alloc_scratch((void**)&rank_o, sizeof(int32_t) * n));
        SKNN_TRY(assign(prev, cid, pdist, nullptr, m, 1, prev_stride));
    }
    k_offsets<<<1, 1024, 0, s>>>(counts, m, out.off, cursor);
    cx.launched();
    unsigned long long* keys;
    SKNN_TRY(cx.alloc_scratch((void**)&keys, sizeof(unsigned long long) * n));
    int sblocks = (int)std::min<int64_t>((n + 255) / 256, 148 * 16);
    k_scatter_keys<<<sblocks, 256, 0, s>>>(cid, pdist, n, out.off, cursor, rank_o, keys);
    cx.launched();
    k_segsort_small<<<m, 256, 0, s>>>(keys, out.off, out.radius);
    cx.launched();
    k_segsort_big<<<m, 1024, 0, s>>>(keys, out.off, out.radius);
    cx.launched();
    int64_t tot = n * (dp / 4);
    int gblocks = (int)std::min<int64_t>((tot + 255) / 256, 148 * 16);
    k_gather_side<<<gblocks, 256, 0, s>>>(keys, Xp, n, dp, out.rows, out.dist, out.orig);
    cx.launched();
    k_side_info<<<(m + 255) / 256, 256, 0, s>>>(out.off, out.radius, out.dist, m, out.tinfo);
    cx.launched();
    return cx.check_launch("build_side");
}

}  // namespace sknn
