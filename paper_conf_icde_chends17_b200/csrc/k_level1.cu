// k_level1.cu -- Step 2 of the method: level-1 (cluster-pair) filtering.
//
// One CTA per query cluster qc fuses the paper's two level-1 kernels:
//   calUB  (§II-C Step 2.1; Fig. 4 calUB/getUBs P:L275-279;
//           GPU version P:L337): pool the bounds r_q + D(qc,tc) + d(c_tc, u_i)
//           over the k members u_i closest to each target center (Eq. 4,
//           Fig. 5) and take the k-th smallest. Each thread keeps a
//           register top-k and stops a cluster early once its bound exceeds
//           its own k-th (the footnote's early termination); the
//           block then selects the k-th smallest among the values that can
//           still matter (<= the smallest per-thread k-th).
//   groupFilter (Alg. 1; Fig. 4 getLB/groupFilter P:L273-277;
//           GPU version P:L339): keep tc iff lb = D - r_q - r_t <= UB
//           (reading R6, plus the R7 rounding slack). Survivors are compacted
//           with warp ballots into shared memory and sorted by (D, tc)
//           ascending -- the candidate order of pointFilter (Fig. 4 line 1,
//           P:L263) -- then written to row qc of the [mq x mt] candidate table.
// B200 design: no atomics in global memory except one counter add per CTA;
// the table row per query cluster removes the paper's atomicAdd append.
#include <cuda_runtime.h>
#include <stdint.h>

#include "sknn_internal.cuh"
#include "sknn_launch.h"

namespace sknn {

typedef unsigned long long u64;

template <int KMAX>
struct RegTopKf {
    float a[KMAX];
    __device__ __forceinline__ void init(int k) {
#pragma unroll
        for (int i = 0; i < KMAX; ++i) a[i] = (i < KMAX - k) ? -1.f : __int_as_float(0x7f800000);
    }
    __device__ __forceinline__ void insert(float v) {
#pragma unroll
        for (int i = KMAX - 1; i > 0; --i) {
            float lo = a[i - 1], cur = a[i];
            a[i] = (v < lo) ? lo : fminf(v, cur);
        }
        a[0] = fminf(a[0], v);
    }
};

__device__ __forceinline__ void cmpx64(u64* s, int i, int p) {
    u64 a = s[i], b = s[p];
    if (b < a) { s[i] = b; s[p] = a; }
}
__device__ __forceinline__ void cmpxf(float* s, int i, int p) {
    float a = s[i], b = s[p];
    if (b < a) { s[i] = b; s[p] = a; }
}

// ascending bitonic (flip + half-cleaner form) over S (power of two) entries
template <typename T, typename F>
__device__ void block_sort_pow2(T* s, int S, F cx) {
    for (int k = 2; k <= S; k <<= 1) {
        for (int t = threadIdx.x; t < S / 2; t += blockDim.x) {
            int blk = t / (k / 2), r = t % (k / 2);
            cx(s, blk * k + r, blk * k + k - 1 - r);
        }
        __syncthreads();
        for (int j = k / 4; j > 0; j >>= 1) {
            for (int t = threadIdx.x; t < S / 2; t += blockDim.x) {
                int i = (t / j) * 2 * j + (t % j);
                cx(s, i, i + j);
            }
            __syncthreads();
        }
    }
}

constexpr int kL1Threads = 256;

template <int KMAX>
__global__ void __launch_bounds__(kL1Threads) k_level1(
    const float* __restrict__ qcent, const float* __restrict__ qrad, const int32_t* __restrict__ qoff,
    const float* __restrict__ tcent, const float* __restrict__ trad, const int32_t* __restrict__ toff,
    const float* __restrict__ tdist, int mt, int dp, int k, float eta, int keys_cap, int shard_rank,
    int shard_count, float* __restrict__ ub_out, int32_t* __restrict__ cand, int32_t* __restrict__ cand_count,
    unsigned long long* __restrict__ cand_pairs) {
    extern __shared__ __align__(16) unsigned char smem[];
    u64* s_keys = reinterpret_cast<u64*>(smem);                      // keys_cap entries
    float* s_vals = reinterpret_cast<float*>(smem);                  // aliases s_keys in phase 1
    float* s_qc = reinterpret_cast<float*>(smem + sizeof(u64) * keys_cap);
    __shared__ int s_cnt;
    __shared__ float s_red[kL1Threads / 32];
    __shared__ float s_ub;

    const int qc = blockIdx.x;
    const int qsize = qoff[qc + 1] - qoff[qc];
    if (qsize == 0 || (shard_count > 1 && qc % shard_count != shard_rank)) {
        if (threadIdx.x == 0) { ub_out[qc] = 0.f; cand_count[qc] = 0; }
        return;
    }
    for (int i = threadIdx.x; i < dp; i += blockDim.x) s_qc[i] = qcent[(int64_t)qc * dp + i];
    if (threadIdx.x == 0) s_cnt = 0;
    __syncthreads();
    const float rq = qrad[qc];
    const float INF = __int_as_float(0x7f800000);

    // ---- phase 1: calUB ----
    RegTopKf<KMAX> top;
    top.init(k);
    for (int tc = threadIdx.x; tc < mt; tc += blockDim.x) {
        int lo = toff[tc], hi = toff[tc + 1];
        if (lo == hi) continue;
        float D = __fsqrt_rn(d2_rows(s_qc, tcent + (int64_t)tc * dp, dp));
        float base = rq + D;
        int cnt = min(k, hi - lo);
        for (int i = 0; i < cnt; ++i) {
            float v = base + __ldg(tdist + hi - 1 - i);   // members closest to the center
            if (!(v < top.a[KMAX - 1])) break;            // early termination
            top.insert(v);
        }
    }
    // T0 = min over threads of their k-th bound: the block k-th is <= T0
    float my = top.a[KMAX - 1];
    for (int o = 16; o > 0; o >>= 1) my = fminf(my, __shfl_xor_sync(0xffffffffu, my, o));
    if ((threadIdx.x & 31) == 0) s_red[threadIdx.x >> 5] = my;
    __syncthreads();
    float T0 = s_red[0];
    for (int w = 1; w < kL1Threads / 32; ++w) T0 = fminf(T0, s_red[w]);
#pragma unroll
    for (int i = 0; i < KMAX; ++i) {
        float v = top.a[i];
        if (v >= 0.f && v <= T0) {
            int pos = atomicAdd(&s_cnt, 1);
            s_vals[pos] = v;
        }
    }
    __syncthreads();
    int nv = s_cnt;
    int S = 1;
    while (S < nv) S <<= 1;
    for (int i = nv + threadIdx.x; i < S; i += blockDim.x) s_vals[i] = INF;
    __syncthreads();
    block_sort_pow2(s_vals, S, cmpxf);
    if (threadIdx.x == 0) {
        float ub = (k - 1 < nv) ? s_vals[k - 1] : INF;
        ub = __fmul_ru(ub, 1.f + 2.f * eta);  // R7: covers rounding of the three summed distances
        s_ub = ub;
        ub_out[qc] = ub;
        s_cnt = 0;
    }
    __syncthreads();
    const float UB = s_ub;

    // ---- phase 2: groupFilter (Alg. 1) ----
    for (int base = 0; base < mt; base += blockDim.x) {
        int tc = base + threadIdx.x;
        bool keep = false;
        float D = 0.f;
        if (tc < mt && toff[tc] != toff[tc + 1]) {
            D = __fsqrt_rn(d2_rows(s_qc, tcent + (int64_t)tc * dp, dp));
            float rt = trad[tc];
            float lb = D - rq - rt;                              // getLB (Eq. 3)
            keep = ti_keep(lb, UB, D + rq + rt, eta);             // Alg. 1 line 4 (R6, R7)
        }
        unsigned m = __ballot_sync(0xffffffffu, keep);
        int wbase = 0;
        if ((threadIdx.x & 31) == 0 && m) wbase = atomicAdd(&s_cnt, __popc(m));
        wbase = __shfl_sync(0xffffffffu, wbase, 0);
        if (keep) {
            int pos = wbase + __popc(m & ((1u << (threadIdx.x & 31)) - 1u));
            s_keys[pos] = (u64(__float_as_uint(D)) << 32) | u64(uint32_t(tc));
        }
    }
    __syncthreads();
    int nc = s_cnt;
    S = 1;
    while (S < nc) S <<= 1;
    for (int i = nc + threadIdx.x; i < S; i += blockDim.x) s_keys[i] = ~0ull;
    __syncthreads();
    block_sort_pow2(s_keys, S, cmpx64);
    int32_t* row = cand + (int64_t)qc * mt;
    for (int i = threadIdx.x; i < nc; i += blockDim.x) row[i] = int32_t(uint32_t(s_keys[i] & 0xffffffffu));
    if (threadIdx.x == 0) {
        cand_count[qc] = nc;
        if (cand_pairs) atomicAdd(cand_pairs, (unsigned long long)nc);
    }
}

sknn_status run_level1(Ctx& cx, const Side& qs, const Side& ts, int k, float eta, int shard_rank, int shard_count,
                       Level1& out, unsigned long long* cand_pairs_counter) {
    const int mq = qs.m, mt = ts.m, dp = ts.dp;
    SKNN_TRY(cx.alloc_scratch((void**)&out.ub, sizeof(float) * mq));
    SKNN_TRY(cx.alloc_scratch((void**)&out.cand, sizeof(int32_t) * (size_t)mq * mt));
    SKNN_TRY(cx.alloc_scratch((void**)&out.cand_count, sizeof(int32_t) * mq));
    int kmax = k <= 8 ? 8 : k <= 16 ? 16 : k <= 24 ? 24 : 32;
    int cap = 1;
    while (cap < mt) cap <<= 1;
    cap = std::max(cap, 4096);  // phase 1 sorts up to 256*32 floats (32 KB) aliasing the key buffer
    size_t smem = sizeof(u64) * cap + sizeof(float) * dp;
    if (smem > 200 * 1024) {
        set_last_error("level-1: too many target clusters for the shared-memory candidate sort");
        return SKNN_ERR_UNSUPPORTED;
    }
#define SKNN_L1(KM)                                                                                           \
    do {                                                                                                      \
        SKNN_CUDA(cudaFuncSetAttribute(k_level1<KM>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem)); \
        k_level1<KM><<<mq, kL1Threads, smem, cx.stream>>>(qs.centers, qs.radius, qs.off, ts.centers, ts.radius, \
                                                          ts.off, ts.dist, mt, dp, k, eta, cap, shard_rank,     \
                                                          shard_count, out.ub,       \
                                                          out.cand, out.cand_count, cand_pairs_counter);      \
    } while (0)
    switch (kmax) {
        case 8: SKNN_L1(8); break;
        case 16: SKNN_L1(16); break;
        case 24: SKNN_L1(24); break;
        default: SKNN_L1(32); break;
    }
#undef SKNN_L1
    cx.launched();
    return cx.check_launch("level1");
}

}  // namespace sknn
