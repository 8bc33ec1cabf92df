// k_dense.cu -- the elastic switch's dense-tile branch (
// the paper's partial level-2 filter idea: when a cluster pair is
// dense, regularity beats per-point TI checks).
//
// For a tile of up to 128 queries of one query cluster and each of its dense
// candidate target clusters, the whole target cluster (no per-point TI checks:
// the regular path of the elastic switch) is streamed through shared memory in
// chunks of NCH targets and the 128 x NCH dot products run on the
// 5th-generation tensor cores:
//
//   a = q - c_r, b = t - c_r            (c_r = query-cluster center rounded to
//                                        integers: re-centring avoids the
//                                        ||q||^2 + ||t||^2 - 2 q.t cancellation)
//   a = a_hi + a_lo (bf16 split), same for b
//   D = a_hi.b_hi + a_hi.b_lo + a_lo.b_hi   tcgen05.mma kind::f16, fp32 accumulator in TMEM
//   d2~ = ||a||^2 + ||b||^2 - 2 D            (lo terms skipped when every lo is 0)
//
// The epilogue (one thread per TMEM lane = query row, tcgen05.ld) is a SCREEN:
// d2~ has a rigorous error bound E = eps (||a||^2 + ||b||^2) + (K+2) 2^-23 d2_k,
// eps = 2^-12 max(1, K/128) (bf16 split truncation 3*2^-16 + fp32 accumulation
// of 3K terms, doubled). A target survives iff d2~ - E <= the row's k-th
// squared distance; survivors are recomputed with the exact fp32 formula every
// path shares (d2_rows) and inserted into the row's register top-k, so the
// result keys are bit-identical to the sparse path's. The per-row top-k is
// handed to the sparse scan, which continues over the remaining (sparse)
// candidate clusters.
//
// Operands use the UMMA canonical K-major SWIZZLE_NONE layout: 8-row x 16-byte
// core matrices; LBO = 128 B (next 8 K-elements), SBO = KP*16 B (next 8 rows).
#include <cuda_bf16.h>
#include <cuda_runtime.h>
#include <stdint.h>

#include "k_scan_common.cuh"

namespace sknn {

struct DenseArgs {
    const float* qrows;
    const int32_t* qoff;
    const float* qcent;
    const float* trows;
    const float* tdist;
    const int32_t* torig;
    const int32_t* toff;
    const float* tcent;
    const float* ub;
    const int32_t* dcand;
    const int32_t* dcount;
    const int2* tiles;
    const int* ntiles;
    int* counter;
    int mt;
    int dp;
    int kp;       // K padded to a multiple of 16 (bf16 MMA K)
    int k;
    float eta;
    float eps_tc;
    key_t* topk_out;  // [n_q x k] in permuted query order
    Counters* counters;
};

constexpr int kDenseM = 128;

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

__device__ __forceinline__ uint64_t umma_desc(uint32_t saddr, uint32_t lbo, uint32_t sbo) {
    uint64_t d = 0;
    d |= (uint64_t)((saddr >> 4) & 0x3FFFu);
    d |= (uint64_t)((lbo >> 4) & 0x3FFFu) << 16;
    d |= (uint64_t)((sbo >> 4) & 0x3FFFu) << 32;
    d |= (uint64_t)1 << 46;  // descriptor version 1 (sm_100); base offset 0; SWIZZLE_NONE
    return d;
}

// kind::f16 instruction descriptor: BF16 x BF16 -> F32, both K-major, M = 128
__host__ __device__ constexpr uint32_t umma_idesc_bf16(int n) {
    return (1u << 4) | (1u << 7) | (1u << 10) | (uint32_t(n >> 3) << 17) | (uint32_t(kDenseM >> 4) << 24);
}

__device__ __forceinline__ void umma_bf16(uint32_t tmem_d, uint64_t a, uint64_t b, uint32_t idesc, uint32_t acc) {
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "setp.ne.b32 p, %4, 0;\n\t"
        "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}\n" ::"r"(tmem_d),
        "l"(a), "l"(b), "r"(idesc), "r"(acc));
}

__device__ __forceinline__ void umma_commit(uint64_t* bar) {
    asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(smem_u32(bar))
                 : "memory");
}

__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t phase) {
    asm volatile(
        "{\n\t.reg .pred P1;\n\t"
        "WAIT_%=:\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n\t"
        "@!P1 bra WAIT_%=;\n\t}\n" ::"r"(smem_u32(bar)),
        "r"(phase)
        : "memory");
}

__device__ __forceinline__ void tmem_ld32(uint32_t taddr, uint32_t (&r)[32]) {
    asm volatile(
        "tcgen05.ld.sync.aligned.32x32b.x32.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,"
        "%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];"
        : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),
          "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15]),
          "=r"(r[16]), "=r"(r[17]), "=r"(r[18]), "=r"(r[19]), "=r"(r[20]), "=r"(r[21]), "=r"(r[22]), "=r"(r[23]),
          "=r"(r[24]), "=r"(r[25]), "=r"(r[26]), "=r"(r[27]), "=r"(r[28]), "=r"(r[29]), "=r"(r[30]), "=r"(r[31])
        : "r"(taddr));
    asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
}

__device__ __forceinline__ void fence_async_smem() { asm volatile("fence.proxy.async.shared::cta;" ::: "memory"); }
__device__ __forceinline__ void tc_fence_before() { asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void tc_fence_after() { asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory"); }

// 8 fp32 -> (hi, lo) bf16 pairs packed as two 16-byte core-matrix rows
__device__ __forceinline__ bool split8(const float (&v)[8], uint4& hi, uint4& lo) {
    uint32_t h[4], l[4];
    bool nz = false;
#pragma unroll
    for (int i = 0; i < 4; ++i) {
        __nv_bfloat16 h0 = __float2bfloat16_rn(v[2 * i]), h1 = __float2bfloat16_rn(v[2 * i + 1]);
        __nv_bfloat16 l0 = __float2bfloat16_rn(v[2 * i] - __bfloat162float(h0));
        __nv_bfloat16 l1 = __float2bfloat16_rn(v[2 * i + 1] - __bfloat162float(h1));
        h[i] = (uint32_t)__bfloat16_as_ushort(h0) | ((uint32_t)__bfloat16_as_ushort(h1) << 16);
        l[i] = (uint32_t)__bfloat16_as_ushort(l0) | ((uint32_t)__bfloat16_as_ushort(l1) << 16);
        nz |= (l[i] & 0x7fff7fffu) != 0u;
    }
    hi = make_uint4(h[0], h[1], h[2], h[3]);
    lo = make_uint4(l[0], l[1], l[2], l[3]);
    return nz;
}

template <int KMAX, int NCH>
__global__ void __launch_bounds__(kDenseM, 1) k_dense(DenseArgs a) {
    extern __shared__ __align__(128) unsigned char smem[];
    const int KP = a.kp;
    const int dp = a.dp;
    const uint32_t sbo = (uint32_t)KP * 16u;  // bytes between 8-row groups
    unsigned char* sA_hi = smem;
    unsigned char* sA_lo = sA_hi + (size_t)kDenseM * KP * 2;
    unsigned char* sB_hi = sA_lo + (size_t)kDenseM * KP * 2;
    unsigned char* sB_lo = sB_hi + (size_t)NCH * KP * 2;
    float* s_tn = reinterpret_cast<float*>(sB_lo + (size_t)NCH * KP * 2);  // [NCH]
    float* s_cr = s_tn + NCH;                                             // [KP]
    __shared__ uint64_t s_bar;
    __shared__ uint32_t s_tmem;
    __shared__ int s_tile, s_loA, s_loB;

    const int tid = threadIdx.x, warp = tid >> 5;
    if (warp == 0) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(&s_tmem)),
                     "r"((uint32_t)NCH));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    if (tid == 0) {
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(&s_bar)));
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tmem = s_tmem;
    const uint32_t tmem_row = tmem + ((uint32_t)(warp * 32) << 16);
    uint32_t phase = 0;
    const uint32_t idesc = umma_idesc_bf16(NCH);
    const float INF = __int_as_float(0x7f800000);
    const float rel_k = 1.f + (float)(KP + 2) * 1.1920929e-7f;  // (K+2) 2^-23
    unsigned long long covered = 0, recomputed = 0;

    for (;;) {
        if (tid == 0) s_tile = atomicAdd(a.counter, 1);
        __syncthreads();
        const int tile = s_tile;
        if (tile >= *a.ntiles) break;
        const int2 tl = a.tiles[tile];
        const int qc = tl.x;
        const int qlo = a.qoff[qc], qsz = a.qoff[qc + 1] - qlo;
        const int r = tid;
        const bool active = tl.y + r < qsz;
        const int qpos = qlo + tl.y + (active ? r : 0);
        const float* qrow = a.qrows + (int64_t)qpos * dp;
        // rounded query-cluster center (re-centring point)
        for (int c = tid; c < KP; c += blockDim.x) s_cr[c] = c < dp ? rintf(a.qcent[(int64_t)qc * dp + c]) : 0.f;
        if (tid == 0) s_loA = 0;
        __syncthreads();
        // stage A = q - c_r (hi/lo bf16) in core-matrix layout; ||a||^2 per row
        {
            const int c8n = KP / 8;
            bool nz = false;
            for (int w = tid; w < kDenseM * c8n; w += blockDim.x) {
                const int row = w / c8n, c8 = w % c8n;
                const bool rv = tl.y + row < qsz;
                const float* src = a.qrows + (int64_t)(qlo + tl.y + (rv ? row : 0)) * dp;
                float v[8];
#pragma unroll
                for (int i = 0; i < 8; ++i) {
                    const int kk = c8 * 8 + i;
                    v[i] = (rv && kk < dp) ? src[kk] - s_cr[kk] : 0.f;
                }
                uint4 hi, lo;
                nz |= split8(v, hi, lo);
                const uint32_t off = (uint32_t)(row >> 3) * sbo + (uint32_t)c8 * 128u + (uint32_t)(row & 7) * 16u;
                *reinterpret_cast<uint4*>(sA_hi + off) = hi;
                *reinterpret_cast<uint4*>(sA_lo + off) = lo;
            }
            if (__syncthreads_or(nz) && tid == 0) s_loA = 1;
        }
        float qn = 0.f;
        for (int c = 0; c < dp; ++c) {
            const float x = qrow[c] - s_cr[c];
            qn = __fmaf_rn(x, x, qn);
        }
        RegTopK<KMAX> top;
        top.init(a.k);
        const float ub = a.ub[qc];
        float theta = ub;
        key_t kth = top.kth();
        float kth2 = __fmul_ru(ub, ub);
        float thr = kth2 * rel_k - qn * (1.f - a.eps_tc);
        const int nd = a.dcount[qc];
        const int32_t* dl = a.dcand + (int64_t)qc * a.mt;
        for (int ci = 0; ci < nd; ++ci) {
            const int tc = __ldg(dl + ci);
            const int lo = __ldg(a.toff + tc), hi = __ldg(a.toff + tc + 1);
            // dense pair: the whole target cluster is screened (no per-point TI
            // checks -- the regular tiled path of the elastic switch)
            const int W0 = lo, W1 = hi;
            for (int j0 = W0; j0 < W1; j0 += NCH) {
                const int nb = min(NCH, W1 - j0);
                // stage B = t - c_r and ||b||^2 (1 - eps)
                if (tid == 0) s_loB = 0;
                __syncthreads();
                {
                    // TPR threads per target row; each converts a contiguous K range
                    constexpr int TPR = kDenseM / NCH;
                    const int row = tid / TPR, part = tid % TPR;
                    const int c8n = KP / 8, c8per = c8n / TPR;
                    const bool rv = row < nb;
                    const float4* src4 = reinterpret_cast<const float4*>(a.trows + (int64_t)(j0 + (rv ? row : 0)) * dp);
                    const float4* cr4 = reinterpret_cast<const float4*>(s_cr);
                    bool nz = false;
                    float tn = 0.f;
#pragma unroll 4
                    for (int c8 = part * c8per; c8 < (part + 1) * c8per; ++c8) {
                        float v[8];
#pragma unroll
                        for (int h = 0; h < 2; ++h) {
                            const int k4 = c8 * 2 + h;
                            float4 x = make_float4(0.f, 0.f, 0.f, 0.f);
                            if (rv && k4 * 4 < dp) {
                                const float4 t4 = __ldg(src4 + k4), c4 = cr4[k4];
                                x = make_float4(t4.x - c4.x, t4.y - c4.y, t4.z - c4.z, t4.w - c4.w);
                            }
                            v[4 * h + 0] = x.x; v[4 * h + 1] = x.y; v[4 * h + 2] = x.z; v[4 * h + 3] = x.w;
                            tn = __fmaf_rn(x.x, x.x, tn); tn = __fmaf_rn(x.y, x.y, tn);
                            tn = __fmaf_rn(x.z, x.z, tn); tn = __fmaf_rn(x.w, x.w, tn);
                        }
                        uint4 hi4, lo4;
                        nz |= split8(v, hi4, lo4);
                        const uint32_t off = (uint32_t)(row >> 3) * sbo + (uint32_t)c8 * 128u + (uint32_t)(row & 7) * 16u;
                        *reinterpret_cast<uint4*>(sB_hi + off) = hi4;
                        *reinterpret_cast<uint4*>(sB_lo + off) = lo4;
                    }
#pragma unroll
                    for (int o = 1; o < TPR; o <<= 1) tn += __shfl_xor_sync(0xffffffffu, tn, o);
                    if (part == 0) s_tn[row] = rv ? tn * (1.f - a.eps_tc) : INF;
                    if (__syncthreads_or(nz) && tid == 0) s_loB = 1;
                }
                fence_async_smem();
                __syncthreads();
                if (tid == 0) {
                    tc_fence_after();
                    const bool loA = s_loA != 0, loB = s_loB != 0;
                    const uint32_t aH = smem_u32(sA_hi), aL = smem_u32(sA_lo);
                    const uint32_t bH = smem_u32(sB_hi), bL = smem_u32(sB_lo);
                    for (int s = 0; s < KP / 16; ++s) {
                        const uint32_t ko = (uint32_t)s * 256u;
                        umma_bf16(tmem, umma_desc(aH + ko, 128u, sbo), umma_desc(bH + ko, 128u, sbo), idesc, s > 0);
                        if (loB) umma_bf16(tmem, umma_desc(aH + ko, 128u, sbo), umma_desc(bL + ko, 128u, sbo), idesc, 1);
                        if (loA) umma_bf16(tmem, umma_desc(aL + ko, 128u, sbo), umma_desc(bH + ko, 128u, sbo), idesc, 1);
                    }
                    umma_commit(&s_bar);
                }
                mbar_wait(&s_bar, phase);
                phase ^= 1u;
                tc_fence_after();
                // epilogue: screen d2~ - E against the row's k-th, exact recompute of survivors
#pragma unroll 1
                for (int cb = 0; cb < NCH / 32; ++cb) {
                    uint32_t v[32];
                    tmem_ld32(tmem_row + (uint32_t)(cb * 32), v);
                    if (!active || cb * 32 >= nb) continue;
                    uint32_t mask = 0;
#pragma unroll
                    for (int j = 0; j < 32; ++j) {
                        const float sc = __fmaf_rn(-2.f, __uint_as_float(v[j]), s_tn[cb * 32 + j]);
                        mask |= (sc <= thr ? 1u : 0u) << j;
                    }
                    while (mask) {
                        const int j = __ffs(mask) - 1;
                        mask &= mask - 1;
                        const int jj = j0 + cb * 32 + j;
                        const float d2 = d2_rows(qrow, a.trows + (int64_t)jj * dp, dp);
                        ++recomputed;
                        if (d2 <= key_d2(kth)) {
                            const key_t key = make_key(d2, __ldg(a.torig + jj));
                            if (key < kth) {
                                top.insert(key);
                                kth = top.kth();
                                const float k2 = key_d2(kth);
                                if (k2 < INF) {
                                    theta = fminf(ub, __fsqrt_ru(k2));
                                    kth2 = fminf(kth2, k2);
                                    thr = kth2 * rel_k - qn * (1.f - a.eps_tc);
                                }
                            }
                        }
                    }
                }
                if (active) covered += (unsigned long long)nb;
                tc_fence_before();
                __syncthreads();
            }
        }
        if (active) {
#pragma unroll
            for (int s = 0; s < KMAX; ++s) {
                const int rr = s - (KMAX - a.k);
                if (rr >= 0) a.topk_out[(int64_t)qpos * a.k + rr] = top.a[s];
            }
        }
        __syncthreads();
    }
    add_counter(&a.counters->evals_dense, covered);
    add_counter(&a.counters->dist_recompute, recomputed);
    tc_fence_before();
    __syncthreads();
    if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"((uint32_t)NCH));
}

template <int KMAX, int NCH>
static sknn_status launch_dense_k(Ctx& cx, const DenseArgs& a) {
    const size_t smem = (size_t)kDenseM * a.kp * 4 + (size_t)NCH * a.kp * 4 + sizeof(float) * (NCH + a.kp);
    SKNN_CUDA(cudaFuncSetAttribute(k_dense<KMAX, NCH>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    int per_sm = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_dense<KMAX, NCH>, kDenseM, smem);
    per_sm = std::max(1, std::min(per_sm, 512 / NCH));  // TMEM: NCH columns per CTA, 512 per SM
    k_dense<KMAX, NCH><<<per_sm * cx.num_sms, kDenseM, smem, cx.stream>>>(a);
    cx.launched();
    return cx.check_launch("dense tiles");
}

template <int NCH>
static sknn_status launch_dense_n(Ctx& cx, const DenseArgs& a) {
    if (a.k <= 8) return launch_dense_k<8, NCH>(cx, a);
    if (a.k <= 16) return launch_dense_k<16, NCH>(cx, a);
    if (a.k <= 24) return launch_dense_k<24, NCH>(cx, a);
    return launch_dense_k<32, NCH>(cx, a);
}

int dense_kp(int dp) { return (dp + 15) & ~15; }
bool dense_supported(int dp) { return dense_kp(dp) <= 256; }

sknn_status run_dense(Ctx& cx, const Side& qs, const Side& ts, const Level1& l1, const DenseParams& p) {
    DenseArgs a{};
    a.qrows = qs.rows; a.qoff = qs.off; a.qcent = qs.centers;
    a.trows = ts.rows; a.tdist = ts.dist; a.torig = ts.orig; a.toff = ts.off; a.tcent = ts.centers;
    a.ub = l1.ub; a.dcand = l1.dcand; a.dcount = l1.dcount;
    a.tiles = l1.dtiles; a.ntiles = l1.dntiles; a.counter = l1.dntiles + 1;
    a.mt = ts.m; a.dp = ts.dp; a.kp = dense_kp(ts.dp); a.k = p.k; a.eta = p.eta;
    a.eps_tc = (float)ldexp(1.0, -12) * std::max(1.f, (float)a.kp / 128.f);
    a.topk_out = p.topk_out; a.counters = p.counters;
    if (a.kp <= 64) return launch_dense_n<128>(cx, a);
    return launch_dense_n<64>(cx, a);
}

}  // namespace sknn
