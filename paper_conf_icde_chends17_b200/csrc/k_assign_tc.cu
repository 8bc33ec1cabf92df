// k_assign_tc.cu -- Step 1 assignment screen on the tensor cores (SURVEY §8(a)
// S3: "argmin_c ||x - c|| ... screen: tensor cores"; P:L323-331 assign every
// point to its closest landmark).
//
// The assignment only has to be approximate (reading R9: TI validity needs the
// RECORDED member-center distance to be exact, not the nearest center), so the
// nearest center is chosen from
//     score_j = ||b_j||^2 - 2 a.b_j,   a = x - o, b_j = c_j - o   (o = mean center)
// with a and b rounded to bf16 and the whole score produced by tcgen05.mma
// (kind::f16, M = 128 points x N = 128 centers per MMA, fp32 accumulation):
// K is augmented by two columns, a' = [a, 1, 1], b'_j = [-2 b_j, hi_j, lo_j]
// with hi + lo the bf16 split of ||b_j||^2 (of the rounded b_j), so
// a'.b'_j = ||b_j||^2 - 2 a.b_j and the epilogue is a plain min (one FMNMX per
// score). ||a||^2 is the same for every j and drops out of the argmin. The
// exact fp32 distance to the chosen center (the shared d2 formula) is then
// recomputed.
//
// Data movement: the centers are pre-converted once per pass into the UMMA
// canonical K-major layout (8-row x 16-byte core matrices), chunk by chunk, so a
// CTA streams them with 1-D bulk async copies (cp.async.bulk, the TMA engine)
// into a double-buffered shared-memory ring while the previous chunk's MMA
// result is reduced from TMEM (tcgen05.ld) by the four epilogue warps.
#include <cuda_bf16.h>
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdlib.h>

#include "sknn_internal.cuh"
#include "sknn_launch.h"
#include "tc_ptx.cuh"

namespace sknn {

constexpr int kTcM = 128;   // points per CTA (TMEM lanes)
constexpr int kTcN = 128;   // centers per chunk (TMEM columns per accumulator)

using tc::desc_kmajor;
using tc::smem_u32;
constexpr uint32_t idesc_bf16_m128(int n) { return tc::idesc_bf16(kTcM, n); }

// o = mean of the m centers: one CTA per column, fixed-order tree (deterministic)
__global__ void k_center_mean(const float* __restrict__ centers, int m, int dp, float* __restrict__ o) {
    __shared__ double red[256];
    const int c = blockIdx.x;
    double s = 0.0;
    for (int j = threadIdx.x; j < m; j += blockDim.x) s += centers[(int64_t)j * dp + c];
    red[threadIdx.x] = s;
    __syncthreads();
    for (int w = blockDim.x / 2; w > 0; w >>= 1) {
        if (threadIdx.x < w) red[threadIdx.x] += red[threadIdx.x + w];
        __syncthreads();
    }
    if (threadIdx.x == 0) o[c] = (float)(red[0] / m);
}

// centers -> b' = [-2 (c - o), hi, lo] (bf16) in chunked core-matrix layout,
// hi + lo = ||bf16(c - o)||^2; padding centers get hi = +inf (score +inf)
__global__ void k_centers_to_tc(const float* __restrict__ centers, int m, int mpad, int dp, int kp,
                                const float* __restrict__ o, __nv_bfloat16* __restrict__ out) {
    const int c8n = kp / 8;
    const float INF = __int_as_float(0x7f800000);
    for (int j = blockIdx.x * blockDim.x + threadIdx.x; j < mpad; j += gridDim.x * blockDim.x) {
        float nb = 0.f;
        if (j < m)
            for (int k = 0; k < dp; ++k) {
                const float v = __bfloat162float(__float2bfloat16_rn(centers[(int64_t)j * dp + k] - o[k]));
                nb = __fmaf_rn(v, v, nb);
            }
        const __nv_bfloat16 hi = __float2bfloat16_rn(j < m ? nb : INF);
        const __nv_bfloat16 lo = __float2bfloat16_rn(j < m ? nb - __bfloat162float(hi) : 0.f);
        const int chunk = j / kTcN, r = j % kTcN;
        for (int c8 = 0; c8 < c8n; ++c8) {
            uint32_t h[4];
#pragma unroll
            for (int i = 0; i < 4; ++i) {
                __nv_bfloat16 e[2];
#pragma unroll
                for (int t = 0; t < 2; ++t) {
                    const int k0 = c8 * 8 + 2 * i + t;
                    float v = 0.f;
                    if (j < m && k0 < dp) v = -2.f * __bfloat162float(__float2bfloat16_rn(centers[(int64_t)j * dp + k0] - o[k0]));
                    e[t] = __float2bfloat16_rn(v);  // exact: -2 times a bf16 value
                    if (k0 == dp) e[t] = hi;
                    if (k0 == dp + 1) e[t] = lo;
                }
                h[i] = (uint32_t)__bfloat16_as_ushort(e[0]) | ((uint32_t)__bfloat16_as_ushort(e[1]) << 16);
            }
            const size_t off = (size_t)chunk * kTcN * kp * 2 + (size_t)(r >> 3) * kp * 16 + (size_t)c8 * 128 + (size_t)(r & 7) * 16;
            *reinterpret_cast<uint4*>(reinterpret_cast<unsigned char*>(out) + off) = make_uint4(h[0], h[1], h[2], h[3]);
        }
    }
}

// One CTA = 128 points, 8 warps: warps w and w + 4 read the same 32 TMEM lanes
// (points) and split each chunk's 128 columns in halves. Streams every center
// chunk through a 2-deep bulk-copy ring (a stage is refilled as soon as its
// MMA completed). (Measured and rejected: 256 points per CTA sharing each
// chunk with a warp-specialised producer and up to 6 stages, one CTA per SM
// -- C4 full pass 2.29 -> 2.68 ms, C5 5.21 -> 5.56 ms.)
constexpr int kTcThreads = 256;
constexpr int kTcMaxStages = 6;
__global__ void __launch_bounds__(kTcThreads, 1) k_assign_tc(const float* __restrict__ Xp, int64_t n, int dp, int kp,
                                                       const float* __restrict__ o,
                                                       const __nv_bfloat16* __restrict__ cbf, int m, int nchunks,
                                                       int nstages, const float* __restrict__ centers,
                                                       int32_t* __restrict__ cid_out, float* __restrict__ dist_out,
                                                       long long* __restrict__ sums, const double* __restrict__ fx,
                                                       int32_t* __restrict__ counts, int stride) {
    extern __shared__ __align__(128) unsigned char smem[];
    const uint32_t a_bytes = (uint32_t)kTcM * kp * 2, b_bytes = (uint32_t)kTcN * kp * 2;
    unsigned char* sA = smem;
    auto sB = [&](int b) { return smem + a_bytes + (uint32_t)b * b_bytes; };
    __shared__ __align__(8) uint64_t bar_full[kTcMaxStages], bar_mma[2];
    __shared__ uint32_t s_tmem;
    const int tid = threadIdx.x, warp = tid >> 5;
    const uint32_t sbo = (uint32_t)kp * 16u;

    if (warp == 0) {
        tc::tmem_alloc(&s_tmem, 2u * kTcN);
    }
    if (tid == 0) {
        for (int i = 0; i < nstages; ++i) tc::mbar_init(smem_u32(&bar_full[i]), 1);
        for (int i = 0; i < 2; ++i) tc::mbar_init(smem_u32(&bar_mma[i]), 1);
        tc::mbar_fence_init();
    }
    // stage A = x - o (bf16) for the CTA's 128 points
    const int64_t row0 = (int64_t)blockIdx.x * kTcM;
    {
        const int c8n = kp / 8;
        for (int w = tid; w < kTcM * c8n; w += blockDim.x) {
            const int r = w / c8n, c8 = w % c8n;
            const int64_t i = (row0 + r) * stride;
            uint32_t h[4];
#pragma unroll
            for (int e = 0; e < 4; ++e) {
                float v0 = 0.f, v1 = 0.f;
                const int k0 = c8 * 8 + 2 * e;
                if (i < n && k0 < dp) v0 = Xp[i * dp + k0] - o[k0];
                if (i < n && k0 + 1 < dp) v1 = Xp[i * dp + k0 + 1] - o[k0 + 1];
                if (k0 == dp || k0 == dp + 1) v0 = 1.f;          // a' = [a, 1, 1]
                if (k0 + 1 == dp || k0 + 1 == dp + 1) v1 = 1.f;
                h[e] = (uint32_t)__bfloat16_as_ushort(__float2bfloat16_rn(v0)) |
                       ((uint32_t)__bfloat16_as_ushort(__float2bfloat16_rn(v1)) << 16);
            }
            const uint32_t off = (uint32_t)(r >> 3) * sbo + (uint32_t)c8 * 128u + (uint32_t)(r & 7) * 16u;
            *reinterpret_cast<uint4*>(sA + off) = make_uint4(h[0], h[1], h[2], h[3]);
        }
    }
    tc::fence_proxy_async();  // generic-proxy smem writes -> visible to the tensor core
    tc::fence_before();
    __syncthreads();
    tc::fence_after();
    const uint32_t tmem = s_tmem;
    const uint32_t idesc = idesc_bf16_m128(kTcN);

    auto issue_copy = [&](int chunk, int buf) {  // chunk -> B stage buf
        const uint32_t bar = smem_u32(&bar_full[buf]);
        tc::expect_tx(bar, b_bytes);
        const unsigned char* src = reinterpret_cast<const unsigned char*>(cbf) + (size_t)chunk * b_bytes;
        tc::bulk_g2s(smem_u32(sB(buf)), src, b_bytes, bar);
    };
    auto issue_mma = [&](int stage, int acc) {  // B stage -> accumulator acc
        tc::fence_after();
        const uint32_t aB = smem_u32(sA), bB = smem_u32(sB(stage));
        for (int s = 0; s < kp / 16; ++s)
            tc::mma_bf16(tmem + (uint32_t)(acc * kTcN), desc_kmajor(aB + s * 256u, sbo), desc_kmajor(bB + s * 256u, sbo),
                         idesc, s > 0);
        tc::mma_commit(smem_u32(&bar_mma[acc]));
    };

    // chunk c lives in B stage c % nstages (phase (c / nstages) & 1 of its
    // full barrier) and accumulates into accumulator c & 1
    uint32_t ph_mma[2] = {0, 0};
    if (tid == 0) {
        for (int c = 0; c < nstages && c < nchunks; ++c) issue_copy(c, c);
        tc::mbar_wait(smem_u32(&bar_full[0]), 0);
        issue_mma(0, 0);
    }
    float best = __int_as_float(0x7f800000);
    int bi = 0;
    const int half = warp >> 2;  // columns [64 * half, 64 * half + 64) of every chunk
    const uint32_t trow = tmem + ((uint32_t)((warp & 3) * 32) << 16);
    for (int c = 0; c < nchunks; ++c) {
        const int buf = c & 1;
        // issue the next chunk's MMA as soon as its copy landed (overlaps this epilogue)
        if (tid == 0 && c + 1 < nchunks) {
            const int ns = (c + 1) % nstages;
            tc::mbar_wait(smem_u32(&bar_full[ns]), ((c + 1) / nstages) & 1);
            issue_mma(ns, (c + 1) & 1);
        }
        tc::mbar_wait(smem_u32(&bar_mma[buf]), ph_mma[buf]);
        ph_mma[buf] ^= 1u;
        tc::fence_after();
        // MMA(c) has consumed B stage c % nstages: refill it now with chunk
        // c + nstages (the accumulator `buf` stays busy until the barrier below;
        // MMA(c + 2) is issued only after it)
        if (tid == 0 && c + nstages < nchunks) issue_copy(c + nstages, c % nstages);
        // per 32 columns: the scores (straight from TMEM), their minimum by a
        // min tree (one FMNMX per score) and, only when it beats the running
        // best, the lowest column holding it (a strict running argmin)
        uint32_t v2[2][32];  // both 32-column blocks of this half, one TMEM round trip
        tc::tmem_ld32x2(trow + (uint32_t)(buf * kTcN + half * 64), trow + (uint32_t)(buf * kTcN + half * 64 + 32),
                        v2[0], v2[1]);
#pragma unroll
        for (int cb = 0; cb < 2; ++cb) {
            const int col = half * 64 + cb * 32;
            float sc[32];
#pragma unroll
            for (int j = 0; j < 32; ++j) sc[j] = __uint_as_float(v2[cb][j]);
            const float mn = min_tree<32>(sc);  // 16 three-input FMNMX3 (was 31 FMNMX)
            // the lowest column holding a new best; a warp-uniform branch (the
            // compiler otherwise if-converts the 32-step search and runs it for
            // every block: ncu, 35% of the C5 pass's instructions)
            const bool better = mn < best;
            if (__any_sync(0xffffffffu, better)) {
                if (better) {
                    int jm = 31;
#pragma unroll
                    for (int j = 31; j >= 0; --j) jm = (sc[j] == mn) ? j : jm;
                    best = mn;
                    bi = c * kTcN + col + jm;
                }
            }
        }
        tc::fence_before();
        __syncthreads();  // accumulator `buf` (TMEM) is free again
    }
    // merge the two column halves (the lower column wins ties)
    __shared__ float s_best[kTcM];
    __shared__ int s_bi[kTcM];
    if (half == 1) {
        s_best[tid - kTcM] = best;
        s_bi[tid - kTcM] = bi;
    }
    __syncthreads();
    const int64_t i = (row0 + tid) * stride;
    if (half == 0 && i < n) {
        const float ob = s_best[tid];
        const int obi = s_bi[tid];
        if (ob < best || (ob == best && obi < bi)) bi = obi;
        const float* xr = Xp + i * dp;
        bi = min(bi, m - 1);
        const float d2 = d2_rows(xr, centers + (int64_t)bi * dp, dp);  // exact fp32, shared formula
        if (cid_out) cid_out[i] = bi;
        if (dist_out) dist_out[i] = __fsqrt_rn(d2);
        if (counts) atomicAdd(counts + bi, 1);
        if (sums) fx_accumulate(sums + (int64_t)bi * dp, xr, dp, *fx);
    }
    tc::fence_before();
    __syncthreads();
    if (warp == 0) tc::tmem_dealloc(tmem, 2u * kTcN);
}

// K = dp + 2 augmented columns, padded to the MMA's K step of 16
static int assign_tc_kp(int dp) { return (dp + 2 + 15) & ~15; }
bool assign_tc_supported(int dp) { return dp >= 8 && assign_tc_kp(dp) <= 256; }

sknn_status run_assign_tc(Ctx& cx, const float* Xp, int64_t n, int dp, const float* centers, int m, int32_t* cid,
                          float* dist, long long* sums, const double* fx, int32_t* counts, int stride) {
    const int kp = assign_tc_kp(dp);
    const int nchunks = (m + kTcN - 1) / kTcN;
    const int mpad = nchunks * kTcN;
    float* o;
    __nv_bfloat16* cbf;
    SKNN_TRY(cx.alloc_scratch((void**)&o, sizeof(float) * dp));
    SKNN_TRY(cx.alloc_scratch((void**)&cbf, (size_t)mpad * kp * 2));
    k_center_mean<<<dp, 256, 0, cx.stream>>>(centers, m, dp, o);
    cx.launched();
    k_centers_to_tc<<<(int)std::min<int64_t>((mpad + 255) / 256, 148 * 8), 256, 0, cx.stream>>>(centers, m, mpad, dp, kp,
                                                                                                o, cbf);
    cx.launched();
    // B ring depth: 2 (SKNN_ASSIGN_STAGES = 3..6 for study). Measured: a
    // 6-deep ring (two CTAs per SM still) is SLOWER on C5 (5.3 -> 5.7 ms per
    // full pass): the pass is bound by the epilogue's ALU pipe (ncu: ALU 60%,
    // one FMNMX per score), not by the chunk loads
    const size_t a_bytes = (size_t)kTcM * kp * 2, b_bytes = (size_t)kTcN * kp * 2;
    const char* es = getenv("SKNN_ASSIGN_STAGES");
    const int want = es ? std::max(2, std::min(kTcMaxStages, atoi(es))) : 2;
    const int nstages = (int)std::max<size_t>(2, std::min<size_t>(want, (110 * 1024 - a_bytes) / b_bytes));
    const size_t smem = std::max<size_t>(a_bytes + nstages * b_bytes, 90 * 1024);
    SKNN_CUDA(cudaFuncSetAttribute(k_assign_tc, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    SKNN_CUDA(cudaFuncSetAttribute(k_assign_tc, cudaFuncAttributePreferredSharedMemoryCarveout, 100));
    const int64_t grid = ((n + stride - 1) / stride + kTcM - 1) / kTcM;
    k_assign_tc<<<(unsigned)grid, kTcThreads, smem, cx.stream>>>(Xp, n, dp, kp, o, cbf, m, nchunks, nstages, centers, cid, dist,
                                                          sums, fx, counts, stride);
    cx.launched();
    return cx.check_launch("assign (tensor cores)");
}

}  // namespace sknn
