// k_dense.cu -- the elastic switch's dense-tile branch (
// the paper's "regular" partial level-2 filter idea: when a
// cluster pair is dense, regularity beats per-point TI checks).
//
// For a tile of up to 128 queries of one query cluster and each of its dense
// candidate target clusters, the whole target cluster (no per-point TI checks)
// is streamed in chunks of NCH targets and the 128 x NCH dot products run on
// the 5th-generation tensor cores:
//
//   a = q - o, b = t - o        o = mean target center rounded to integers
//                               (re-centring against ||q||^2 + ||t||^2 - 2 q.t
//                               cancellation; integer data stays integer)
//   a = a_hi + a_lo (bf16 split), same for b
//   D = a_hi.b_hi [+ a_hi.b_lo + a_lo.b_hi]   tcgen05.mma kind::f16, fp32 in TMEM
//   d2~ = ||a||^2 + ||b||^2 - 2 D             (lo terms only when some lo != 0)
//
// B200 data path: both point sets are converted ONCE per join into the UMMA
// canonical K-major SWIZZLE_NONE layout (8-row x 16-byte core matrices; LBO =
// 128 B, SBO = KP*16 B), every cluster starting on an 8-row boundary, so a
// 128-query A tile and every NCH-target B chunk are contiguous byte ranges.
// They move with 1-D bulk async copies (cp.async.bulk, the TMA engine) through
// a 2-deep shared-memory ring, while the MMA of chunk g+1 runs into the second
// TMEM accumulator and the four warps reduce chunk g (tcgen05.ld).
//
// The epilogue (one thread per TMEM lane = query row) is a SCREEN: d2~ has the
// rigorous error bound E = eps (||a||^2 + ||b||^2) + (K+2) 2^-23 d2_k with
// eps = 2^-12 max(1, K/128) (bf16 split truncation + fp32 accumulation of 3K
// terms, doubled). A target survives iff d2~ - E <= the row's k-th squared
// distance; survivors are recomputed with the exact fp32 formula every path
// shares (d2_rows) and inserted into the row's register top-k, so the keys are
// bit-identical to the sparse path's. The sparse scan continues from the
// per-row top-k over the remaining (sparse) candidate clusters.
#include <cuda_bf16.h>
#include <cuda_runtime.h>
#include <math.h>
#include <stdint.h>

#include "k_scan_common.cuh"

namespace sknn {

constexpr int kDenseM = 128;

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

__device__ __forceinline__ uint64_t umma_desc(uint32_t saddr, uint32_t sbo) {
    return (uint64_t)((saddr >> 4) & 0x3FFFu) | ((uint64_t)(128u >> 4) << 16) | ((uint64_t)((sbo >> 4) & 0x3FFFu) << 32) |
           ((uint64_t)1 << 46);  // LBO 128 B, descriptor version 1 (sm_100), SWIZZLE_NONE
}

// kind::f16 instruction descriptor: BF16 x BF16 -> F32, both K-major, M = 128
__host__ __device__ constexpr uint32_t umma_idesc_bf16(int n) {
    return (1u << 4) | (1u << 7) | (1u << 10) | (uint32_t(n >> 3) << 17) | (uint32_t(kDenseM >> 4) << 24);
}

__device__ __forceinline__ void umma_bf16(uint32_t tmem_d, uint64_t a, uint64_t b, uint32_t idesc, uint32_t acc) {
    asm volatile(
        "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
        "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}\n" ::"r"(tmem_d),
        "l"(a), "l"(b), "r"(idesc), "r"(acc));
}

__device__ __forceinline__ void umma_commit(uint32_t bar) {
    asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(bar) : "memory");
}

__device__ __forceinline__ void mbar_wait(uint32_t bar, uint32_t phase) {
    asm volatile(
        "{\n\t.reg .pred P1;\n\tWAIT_%=:\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n\t"
        "@!P1 bra WAIT_%=;\n\t}\n" ::"r"(bar),
        "r"(phase)
        : "memory");
}

__device__ __forceinline__ void bulk_g2s(uint32_t dst, const void* src, uint32_t bytes, uint32_t bar) {
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(dst),
                 "l"(src), "r"(bytes), "r"(bar)
                 : "memory");
}

__device__ __forceinline__ void expect_tx(uint32_t bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(bytes) : "memory");
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

__device__ __forceinline__ void tc_fence_before() { asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void tc_fence_after() { asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory"); }

// ------------------------------------------------------ tile conversion --
// rintf of the mean center: the common origin o of both point sets
__global__ void k_dense_origin(const float* __restrict__ centers, int m, int dp, int kp, float* __restrict__ o) {
    __shared__ double red[256];
    const int c = blockIdx.x;
    double s = 0.0;
    if (c < dp)
        for (int j = threadIdx.x; j < m; j += blockDim.x) s += centers[(int64_t)j * dp + c];
    red[threadIdx.x] = s;
    __syncthreads();
    for (int w = blockDim.x / 2; w > 0; w >>= 1) {
        if (threadIdx.x < w) red[threadIdx.x] += red[threadIdx.x + w];
        __syncthreads();
    }
    if (threadIdx.x == 0) o[c] = c < dp ? rintf((float)(red[0] / m)) : 0.f;
}

// ||c - o|| of every center: the magnitude the dense screen's error bound scales with
__global__ void k_center_dist_o(const float* __restrict__ centers, int m, int dp, const float* __restrict__ o,
                                float* __restrict__ out) {
    for (int c = blockIdx.x * blockDim.x + threadIdx.x; c < m; c += gridDim.x * blockDim.x) {
        float s = 0.f;
        for (int k = 0; k < dp; ++k) {
            const float v = centers[(int64_t)c * dp + k] - o[k];
            s = __fmaf_rn(v, v, s);
        }
        out[c] = sqrtf(s);
    }
}

// cluster sizes rounded up to 8 rows (padded CSR for 8-row-aligned tiles)
__global__ void k_pad8(const int32_t* __restrict__ off, int m, int32_t* __restrict__ cnt8) {
    for (int c = blockIdx.x * blockDim.x + threadIdx.x; c < m; c += gridDim.x * blockDim.x)
        cnt8[c] = ((off[c + 1] - off[c]) + 7) & ~7;
}

// rows (cluster order) -> bf16 hi/lo (x - o) tiles + ||x - o||^2 * nscale, at padded positions
__global__ void __launch_bounds__(256) k_to_tiles(const float* __restrict__ rows, const int32_t* __restrict__ off,
                                                  const int32_t* __restrict__ offp, int dp, int kp,
                                                  const float* __restrict__ o, float nscale,
                                                  __nv_bfloat16* __restrict__ hi, __nv_bfloat16* __restrict__ lo,
                                                  float* __restrict__ norm, float* __restrict__ norm_raw,
                                                  int* __restrict__ lo_flag) {
    const int c = blockIdx.x;
    const int lo0 = off[c], size = off[c + 1] - lo0, p0 = offp[c];
    const int c8n = kp / 8;
    const size_t sbo = (size_t)kp * 16;
    bool nz = false;
    for (int w = threadIdx.x; w < size * c8n; w += blockDim.x) {
        const int r = w / c8n, c8 = w % c8n;
        const float* src = rows + (int64_t)(lo0 + r) * dp;
        uint32_t h[4], l[4];
#pragma unroll
        for (int i = 0; i < 4; ++i) {
            float v[2];
#pragma unroll
            for (int e = 0; e < 2; ++e) {
                const int kk = c8 * 8 + 2 * i + e;
                v[e] = kk < dp ? src[kk] - o[kk] : 0.f;
            }
            const __nv_bfloat16 h0 = __float2bfloat16_rn(v[0]), h1 = __float2bfloat16_rn(v[1]);
            const __nv_bfloat16 l0 = __float2bfloat16_rn(v[0] - __bfloat162float(h0));
            const __nv_bfloat16 l1 = __float2bfloat16_rn(v[1] - __bfloat162float(h1));
            h[i] = (uint32_t)__bfloat16_as_ushort(h0) | ((uint32_t)__bfloat16_as_ushort(h1) << 16);
            l[i] = (uint32_t)__bfloat16_as_ushort(l0) | ((uint32_t)__bfloat16_as_ushort(l1) << 16);
            nz |= (l[i] & 0x7fff7fffu) != 0u;
        }
        const int p = p0 + r;
        const size_t byte = (size_t)(p >> 3) * sbo + (size_t)c8 * 128 + (size_t)(p & 7) * 16;
        *reinterpret_cast<uint4*>(reinterpret_cast<unsigned char*>(hi) + byte) = make_uint4(h[0], h[1], h[2], h[3]);
        *reinterpret_cast<uint4*>(reinterpret_cast<unsigned char*>(lo) + byte) = make_uint4(l[0], l[1], l[2], l[3]);
    }
    for (int r = threadIdx.x; r < size; r += blockDim.x) {
        const float* src = rows + (int64_t)(lo0 + r) * dp;
        float s = 0.f;
        for (int kk = 0; kk < dp; ++kk) {
            const float v = src[kk] - o[kk];
            s = __fmaf_rn(v, v, s);
        }
        norm[p0 + r] = s * nscale;
        if (norm_raw) norm_raw[p0 + r] = s;
    }
    if (__syncthreads_or(nz) && threadIdx.x == 0) atomicOr(lo_flag, 1);
}

__global__ void k_fill_f(float* __restrict__ p, int64_t n, float v) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) p[i] = v;
}

// ----------------------------------------------------------------- kernel --
struct DenseArgs {
    const float* qrows;
    const int32_t* qoff;
    const int32_t* qoffp;
    const unsigned char* qhi;
    const unsigned char* qlo;
    const float* qn;
    const float* trows;
    const int32_t* torig;
    const int32_t* toff;
    const int32_t* toffp;
    const unsigned char* thi;
    const unsigned char* tlo;
    const float* tn;       // ||b||^2 (1 - eps), +inf on padding rows
    const int* lo_flag;    // [2]: query side, target side has a nonzero lo part
    const float* ub;
    const int32_t* dcand;
    const int32_t* dcount;
    const int2* tiles;
    const int* ntiles;
    int* counter;
    int mt;
    int dp;
    int kp;
    int k;
    float eps_tc;
    key_t* topk_out;
    Counters* counters;
};

// per-tile chunk sequence: every dense candidate cluster in NCH-target chunks
template <int NCH>
struct ChunkIter {
    const int32_t* dl;
    int nd, ci, c, nch, tc, size;
    __device__ __forceinline__ void start(const DenseArgs& a, int qc) {
        dl = a.dcand + (int64_t)qc * a.mt;
        nd = a.dcount[qc];
        ci = -1;
        c = 0;
        nch = 0;
        advance(a);
    }
    // moves to the next chunk; false when exhausted
    __device__ __forceinline__ bool advance(const DenseArgs& a) {
        ++c;
        while (c >= nch) {
            if (++ci >= nd) return false;
            tc = __ldg(dl + ci);
            size = __ldg(a.toff + tc + 1) - __ldg(a.toff + tc);
            nch = (size + NCH - 1) / NCH;
            c = 0;
        }
        return true;
    }
    __device__ __forceinline__ bool valid() const { return ci < nd; }
};

template <int KMAX, int NCH>
__global__ void __launch_bounds__(kDenseM, 1) k_dense(DenseArgs a) {
    extern __shared__ __align__(128) unsigned char smem[];
    const int KP = a.kp;
    const int dp = a.dp;
    const uint32_t sbo = (uint32_t)KP * 16u;
    const uint32_t a_bytes = (uint32_t)kDenseM * KP * 2, b_bytes = (uint32_t)NCH * KP * 2;
    // layout: A_hi | A_lo | B_hi[2] | B_lo[2] | tn[2][NCH]
    unsigned char* sA = smem;
    unsigned char* sB = smem + 2 * a_bytes;
    float* s_tn = reinterpret_cast<float*>(sB + 4 * b_bytes);
    __shared__ __align__(8) uint64_t bar_a, bar_full[2], bar_mma[2];
    __shared__ uint32_t s_tmem;
    __shared__ int s_tile;

    const int tid = threadIdx.x, warp = tid >> 5;
    if (warp == 0) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(&s_tmem)),
                     "r"((uint32_t)(2 * NCH)));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    if (tid == 0) {
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(&bar_a)));
        for (int i = 0; i < 2; ++i) {
            asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(&bar_full[i])));
            asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(&bar_mma[i])));
        }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tmem = s_tmem;
    const uint32_t tmem_row = tmem + ((uint32_t)(warp * 32) << 16);
    const uint32_t idesc = umma_idesc_bf16(NCH);
    const bool loA = a.lo_flag[0] != 0, loB = a.lo_flag[1] != 0;
    const uint32_t bstage = loB ? 2 * b_bytes : b_bytes;  // bytes moved per B chunk
    const float INF = __int_as_float(0x7f800000);
    const float rel_k = 1.f + (float)(KP + 2) * 1.1920929e-7f;  // (K+2) 2^-23
    const float qscale = 1.f - a.eps_tc;
    uint32_t ph_a = 0, ph_full[2] = {0, 0}, ph_mma[2] = {0, 0};
    unsigned long long covered = 0, recomputed = 0;

    auto issue_b = [&](const ChunkIter<NCH>& it, int buf) {
        const uint32_t bar = smem_u32(&bar_full[buf]);
        expect_tx(bar, bstage + NCH * 4);
        const size_t p = (size_t)__ldg(a.toffp + it.tc) + (size_t)it.c * NCH;  // 8-aligned padded row
        const size_t byte = (p >> 3) * sbo;
        bulk_g2s(smem_u32(sB + buf * b_bytes), a.thi + byte, b_bytes, bar);
        if (loB) bulk_g2s(smem_u32(sB + (2 + buf) * b_bytes), a.tlo + byte, b_bytes, bar);
        bulk_g2s(smem_u32(s_tn + buf * NCH), a.tn + p, NCH * 4, bar);
    };
    auto issue_mma = [&](int buf) {
        tc_fence_after();
        const uint32_t aH = smem_u32(sA), aL = smem_u32(sA + a_bytes);
        const uint32_t bH = smem_u32(sB + buf * b_bytes), bL = smem_u32(sB + (2 + buf) * b_bytes);
        const uint32_t d = tmem + (uint32_t)(buf * NCH);
        for (int s = 0; s < KP / 16; ++s) {
            const uint32_t ko = (uint32_t)s * 256u;
            umma_bf16(d, umma_desc(aH + ko, sbo), umma_desc(bH + ko, sbo), idesc, s > 0);
            if (loB) umma_bf16(d, umma_desc(aH + ko, sbo), umma_desc(bL + ko, sbo), idesc, 1);
            if (loA) umma_bf16(d, umma_desc(aL + ko, sbo), umma_desc(bH + ko, sbo), idesc, 1);
        }
        umma_commit(smem_u32(&bar_mma[buf]));
    };

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
        const size_t qp = (size_t)a.qoffp[qc] + tl.y;  // padded row of the tile's first query
        ChunkIter<NCH> prod, cons;
        prod.start(a, qc);
        cons.start(a, qc);
        if (tid == 0) {
            const uint32_t bar = smem_u32(&bar_a);
            expect_tx(bar, loA ? 2 * a_bytes : a_bytes);
            bulk_g2s(smem_u32(sA), a.qhi + (qp >> 3) * sbo, a_bytes, bar);
            if (loA) bulk_g2s(smem_u32(sA + a_bytes), a.qlo + (qp >> 3) * sbo, a_bytes, bar);
            if (prod.valid()) {
                issue_b(prod, 0);
                if (prod.advance(a)) issue_b(prod, 1);
                prod.advance(a);  // now two chunks ahead of the consumer
            }
            mbar_wait(smem_u32(&bar_a), ph_a);
            if (cons.valid()) {
                mbar_wait(smem_u32(&bar_full[0]), ph_full[0]);
                issue_mma(0);
            }
        }
        ph_a ^= 1u;
        if (cons.valid()) ph_full[0] ^= 1u;
        const float qn = active ? __ldg(a.qn + qp + r) : 0.f;
        RegTopK<KMAX> top;
        top.init(a.k);
        key_t kth = top.kth();
        const float ub = a.ub[qc];
        float kth2 = __fmul_ru(ub, ub);
        float thr = kth2 * rel_k - qn * qscale;
        for (int g = 0; cons.valid(); ++g) {
            const int buf = g & 1;
            // next chunk's MMA goes into the other accumulator while this one is reduced
            ChunkIter<NCH> nxt = cons;
            const bool has_next = nxt.advance(a);
            if (tid == 0 && has_next) {
                mbar_wait(smem_u32(&bar_full[buf ^ 1]), ph_full[buf ^ 1]);
                issue_mma(buf ^ 1);
            }
            if (has_next) ph_full[buf ^ 1] ^= 1u;
            mbar_wait(smem_u32(&bar_mma[buf]), ph_mma[buf]);
            ph_mma[buf] ^= 1u;
            tc_fence_after();
            const int nb = min(NCH, cons.size - cons.c * NCH);
            const int j0 = __ldg(a.toff + cons.tc) + cons.c * NCH;  // real (unpadded) first target
            const float* tnv = s_tn + buf * NCH;
#pragma unroll 1
            for (int cb = 0; cb < NCH / 32; ++cb) {
                uint32_t v[32];
                tmem_ld32(tmem_row + (uint32_t)(buf * NCH + cb * 32), v);
                if (!active || cb * 32 >= nb) continue;
                uint32_t mask = 0;
#pragma unroll
                for (int j = 0; j < 32; ++j) {
                    const float sc = __fmaf_rn(-2.f, __uint_as_float(v[j]), tnv[cb * 32 + j]);
                    mask |= (sc <= thr ? 1u : 0u) << j;
                }
                if (cb * 32 + 32 > nb) mask &= (1u << (nb - cb * 32)) - 1u;
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
                            if (k2 < kth2) {
                                kth2 = k2;
                                thr = kth2 * rel_k - qn * qscale;
                            }
                        }
                    }
                }
            }
            if (active) covered += (unsigned long long)nb;
            tc_fence_before();
            __syncthreads();  // stage `buf` (smem) and accumulator `buf` (TMEM) are free
            if (tid == 0 && prod.valid()) {
                issue_b(prod, buf);
                prod.advance(a);
            }
            cons = nxt;
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
    if (warp == 0)
        asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"((uint32_t)(2 * NCH)));
}

template <int KMAX, int NCH>
static sknn_status launch_dense_k(Ctx& cx, const DenseArgs& a) {
    const size_t smem = 2 * (size_t)kDenseM * a.kp * 2 + 4 * (size_t)NCH * a.kp * 2 + 2 * NCH * 4;
    SKNN_CUDA(cudaFuncSetAttribute(k_dense<KMAX, NCH>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    int per_sm = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_dense<KMAX, NCH>, kDenseM, smem);
    per_sm = std::max(1, std::min(per_sm, 512 / (2 * NCH)));  // TMEM: 2*NCH columns per CTA
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

// Converted tile set of one side: padded CSR + bf16 hi/lo + norms
// (scaled by 1 - eps for the target role, raw for the query role).
struct DenseSide {
    int32_t* offp = nullptr;
    unsigned char* hi = nullptr;
    unsigned char* lo = nullptr;
    float* norm = nullptr;
    float* norm_raw = nullptr;
};

static sknn_status convert_side(Ctx& cx, const Side& sd, int kp, const float* o, float nscale, bool want_raw,
                                int* lo_flag, DenseSide& out) {
    const int m = sd.m;
    int32_t* cnt8;
    SKNN_TRY(cx.alloc_scratch((void**)&out.offp, sizeof(int32_t) * (m + 1)));
    SKNN_TRY(cx.alloc_scratch((void**)&cnt8, sizeof(int32_t) * 2 * m));
    int32_t* dummy = cnt8 + m;
    k_pad8<<<std::max(1, std::min((m + 255) / 256, 148 * 4)), 256, 0, cx.stream>>>(sd.off, m, cnt8);
    cx.launched();
    k_offsets<<<1, 1024, 0, cx.stream>>>(cnt8, m, out.offp, dummy);
    cx.launched();
    // upper bound of padded rows + a guard for the 128-row tile over-read
    const int64_t npad = sd.n + 7LL * m + 256;
    const size_t tile_bytes = (size_t)npad * kp * 2;
    SKNN_TRY(cx.alloc_scratch((void**)&out.hi, tile_bytes));
    SKNN_TRY(cx.alloc_scratch((void**)&out.lo, tile_bytes));
    SKNN_TRY(cx.alloc_scratch((void**)&out.norm, sizeof(float) * npad));
    if (want_raw) SKNN_TRY(cx.alloc_scratch((void**)&out.norm_raw, sizeof(float) * npad));
    SKNN_CUDA(cudaMemsetAsync(out.hi, 0, tile_bytes, cx.stream));
    SKNN_CUDA(cudaMemsetAsync(out.lo, 0, tile_bytes, cx.stream));
    const int fb = (int)std::min<int64_t>((npad + 255) / 256, 148 * 8);
    k_fill_f<<<fb, 256, 0, cx.stream>>>(out.norm, npad, INFINITY);
    cx.launched();
    if (want_raw) {
        k_fill_f<<<fb, 256, 0, cx.stream>>>(out.norm_raw, npad, 0.f);
        cx.launched();
    }
    k_to_tiles<<<m, 256, 0, cx.stream>>>(sd.rows, sd.off, out.offp, sd.dp, kp, o, nscale,
                                        reinterpret_cast<__nv_bfloat16*>(out.hi),
                                        reinterpret_cast<__nv_bfloat16*>(out.lo), out.norm, out.norm_raw, lo_flag);
    cx.launched();
    return cx.check_launch("dense tile conversion");
}

float dense_eps(int dp) { return (float)ldexp(1.0, -12) * std::max(1.f, (float)dense_kp(dp) / 128.f); }

// common origin o (rounded mean target center) and ||c - o|| per cluster of both sides
sknn_status dense_prepare(Ctx& cx, const Side& qs, const Side& ts, DenseOrigin& out) {
    const int kp = dense_kp(ts.dp);
    SKNN_TRY(cx.alloc_scratch((void**)&out.o, sizeof(float) * kp));
    SKNN_TRY(cx.alloc_scratch((void**)&out.ct_o, sizeof(float) * ts.m));
    k_dense_origin<<<kp, 256, 0, cx.stream>>>(ts.centers, ts.m, ts.dp, kp, out.o);
    cx.launched();
    k_center_dist_o<<<(ts.m + 255) / 256, 256, 0, cx.stream>>>(ts.centers, ts.m, ts.dp, out.o, out.ct_o);
    cx.launched();
    if (&qs == &ts) {
        out.cq_o = out.ct_o;
    } else {
        SKNN_TRY(cx.alloc_scratch((void**)&out.cq_o, sizeof(float) * qs.m));
        k_center_dist_o<<<(qs.m + 255) / 256, 256, 0, cx.stream>>>(qs.centers, qs.m, qs.dp, out.o, out.cq_o);
        cx.launched();
    }
    out.eps = dense_eps(ts.dp);
    return cx.check_launch("dense origin");
}

sknn_status run_dense(Ctx& cx, const Side& qs, const Side& ts, const Level1& l1, const DenseParams& p) {
    const int kp = dense_kp(ts.dp);
    const float eps_tc = dense_eps(ts.dp);
    const bool self = &qs == &ts;
    const float* o = p.origin;
    int* lo_flag;
    SKNN_TRY(cx.alloc_scratch((void**)&lo_flag, sizeof(int) * 2));
    SKNN_CUDA(cudaMemsetAsync(lo_flag, 0, sizeof(int) * 2, cx.stream));
    DenseSide tq, tt;
    SKNN_TRY(convert_side(cx, ts, kp, o, 1.f - eps_tc, self, lo_flag + 1, tt));
    if (self) {
        tq = tt;
        tq.norm = tt.norm_raw;
        SKNN_CUDA(cudaMemcpyAsync(lo_flag, lo_flag + 1, sizeof(int), cudaMemcpyDeviceToDevice, cx.stream));
    } else {
        SKNN_TRY(convert_side(cx, qs, kp, o, 1.f, false, lo_flag, tq));
    }
    DenseArgs a{};
    a.qrows = qs.rows; a.qoff = qs.off; a.qoffp = tq.offp; a.qhi = tq.hi; a.qlo = tq.lo; a.qn = tq.norm;
    a.trows = ts.rows; a.torig = ts.orig; a.toff = ts.off; a.toffp = tt.offp; a.thi = tt.hi; a.tlo = tt.lo;
    a.tn = tt.norm; a.lo_flag = lo_flag;
    a.ub = l1.ub; a.dcand = l1.dcand; a.dcount = l1.dcount;
    a.tiles = l1.dtiles; a.ntiles = l1.dntiles; a.counter = l1.dntiles + 1;
    a.mt = ts.m; a.dp = ts.dp; a.kp = kp; a.k = p.k; a.eps_tc = eps_tc;
    a.topk_out = p.topk_out; a.counters = p.counters;
    if (kp <= 64) return launch_dense_n<128>(cx, a);
    return launch_dense_n<64>(cx, a);
}

}  // namespace sknn
