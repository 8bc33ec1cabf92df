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
#include <stdlib.h>
#include <stdint.h>

#include "k_scan_common.cuh"
#include "tc_ptx.cuh"

namespace sknn {

constexpr int kDenseM = 128;

using tc::smem_u32;
using tc::mbar_wait;
using tc::bulk_g2s;
using tc::expect_tx;
using tc::tmem_ld32;
using tc::fence_before;
using tc::fence_after;
__device__ __forceinline__ uint64_t umma_desc(uint32_t saddr, uint32_t sbo) { return tc::desc_kmajor(saddr, sbo); }
__host__ __device__ constexpr uint32_t umma_idesc_bf16(int n) { return tc::idesc_bf16(kDenseM, n); }

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
                                                  int* __restrict__ lo_flag, int* __restrict__ amax_flag) {
    const int c = blockIdx.x;
    const int lo0 = off[c], size = off[c + 1] - lo0, p0 = offp[c];
    const int c8n = kp / 8;
    const size_t sbo = (size_t)kp * 16;
    bool nz = false;
    float amax = 0.f;  // max |x - o| over the side (exact-path test)
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
                amax = fmaxf(amax, fabsf(v[e]));
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
    for (int o = 16; o > 0; o >>= 1) amax = fmaxf(amax, __shfl_xor_sync(0xffffffffu, amax, o));
    if ((threadIdx.x & 31) == 0 && amax > 0.f) atomicMax(amax_flag, __float_as_int(amax));  // >= 0: int order
}

// self-join: the query side's flags are the target side's
__global__ void k_copy_flags(int* f) {
    if (threadIdx.x == 0) {
        f[0] = f[1];
        f[2] = f[3];
    }
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
    const int* lo_flag;    // [4]: query side, target side has a nonzero lo part; max |x - o| bits of each side
    const float* tn_raw;   // ||b||^2 unscaled, +inf on padding rows (exact variant)
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
    // the chunks of each dense candidate cluster are visited LAST first: the
    // members are stored by distance to their center descending (R11), so
    // the tail holds the members nearest the center, which for most queries
    // of a near cluster are the near targets -- the k-th distance tightens
    // early and far fewer keys enter the top-k (measured: C4 dense stage)
    const int32_t* dl;
    int nd, ci, c, r, nch, tc, size;
    __device__ __forceinline__ void start(const DenseArgs& a, int qc) {
        dl = a.dcand + (int64_t)qc * a.mt;
        nd = a.dcount[qc];
        ci = -1;
        r = 0;
        nch = 0;
        advance(a);
    }
    // moves to the next chunk; false when exhausted
    __device__ __forceinline__ bool advance(const DenseArgs& a) {
        ++r;
        while (r >= nch) {
            if (++ci >= nd) return false;
            tc = __ldg(dl + ci);
            size = __ldg(a.toff + tc + 1) - __ldg(a.toff + tc);
            nch = (size + NCH - 1) / NCH;
            r = 0;
        }
        c = nch - 1 - r;
        return true;
    }
    __device__ __forceinline__ bool valid() const { return ci < nd; }
};

// Exact integer tiles: when neither side has a nonzero bf16 lo part (the
// re-centred coordinates are integers |x - o| <= 256, exact in bf16) and
// dp (A + B)^2 < 2^24 (A, B = max |x - o| per side), every product and every
// partial sum of a.b, ||a||^2 and ||b||^2 is an integer below 2^24, so the
// fp32 MMA result and d2 = ||a||^2 + ||b||^2 - 2 a.b are EXACT and equal the
// shared SIMT formula's d2 bit for bit: no screen slack, no recompute.
__device__ __forceinline__ bool dense_exact_ok(const int* flags, int dp) {
    if (flags[0] | flags[1]) return false;
    const double s = (double)__int_as_float(flags[2]) + (double)__int_as_float(flags[3]);
    return (double)dp * s * s < 16777216.0;
}

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

    if (dense_exact_ok(a.lo_flag, a.dp)) return;  // k_dense_exact handles this join
    const int tid = threadIdx.x, warp = tid >> 5;
    if (warp == 0) {
        tc::tmem_alloc(&s_tmem, (uint32_t)(2 * NCH));
    }
    if (tid == 0) {
        tc::mbar_init(smem_u32(&bar_a), 1);
        for (int i = 0; i < 2; ++i) {
            tc::mbar_init(smem_u32(&bar_full[i]), 1);
            tc::mbar_init(smem_u32(&bar_mma[i]), 1);
        }
        tc::mbar_fence_init();
    }
    fence_before();
    __syncthreads();
    fence_after();
    const uint32_t tmem = s_tmem;
    const uint32_t tmem_row = tmem + ((uint32_t)(warp * 32) << 16);
    const uint32_t idesc = umma_idesc_bf16(NCH);
    const bool loA = a.lo_flag[0] != 0, loB = a.lo_flag[1] != 0;
    if (blockIdx.x == 0 && threadIdx.x == 0) atomicMax(&a.counters->dense_terms, 1ull + loA + loB);
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
        fence_after();
        const uint32_t aH = smem_u32(sA), aL = smem_u32(sA + a_bytes);
        const uint32_t bH = smem_u32(sB + buf * b_bytes), bL = smem_u32(sB + (2 + buf) * b_bytes);
        const uint32_t d = tmem + (uint32_t)(buf * NCH);
        for (int s = 0; s < KP / 16; ++s) {
            const uint32_t ko = (uint32_t)s * 256u;
            tc::mma_bf16(d, umma_desc(aH + ko, sbo), umma_desc(bH + ko, sbo), idesc, s > 0);
            if (loB) tc::mma_bf16(d, umma_desc(aH + ko, sbo), umma_desc(bL + ko, sbo), idesc, 1);
            if (loA) tc::mma_bf16(d, umma_desc(aL + ko, sbo), umma_desc(bH + ko, sbo), idesc, 1);
        }
        tc::mma_commit(smem_u32(&bar_mma[buf]));
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
            fence_after();
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
                    const int j = 31 - __clz(mask);  // highest column first (nearer the center)
                    mask &= ~(1u << j);
                    const int jj = j0 + cb * 32 + j;
                    const float d2 = d2_rows(qrow, a.trows + (int64_t)jj * dp, dp);
                    ++recomputed;
                    if (d2 <= key_d2(kth)) {
                        const key_t key = make_key(d2, __ldg(a.torig + jj));
                        if (key_lt(key, kth)) {
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
            fence_before();
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
    fence_before();
    __syncthreads();
    if (warp == 0)
        tc::tmem_dealloc(tmem, (uint32_t)(2 * NCH));
}

// ------------------------------------------------------ exact dense tiles --
// Warp-specialised: warp 8 (one elected thread) is the producer -- tile
// scheduler, bulk copies of the A tile (128 queries) and of the NCH-target B
// chunks through a kExStages ring, tcgen05.mma of each chunk into one of
// kExAcc TMEM accumulators; warps 0-7 are the epilogue -- two threads per query
// row (TMEM lanes 32 (w % 4) .. + 31), each over one half of the chunk's
// columns, with its own register top-k; the two halves share their k-th
// distance through shared memory (the smaller of two subsets' k-th distances
// is still >= the row's true k-th) and are merged when the tile ends.
// Barriers: full[s] (chunk landed), sfree[s] (its MMA done: stage reusable),
// mma[c] (accumulator ready), afree[c] (epilogue done with it: count 8 warps),
// tfull/tfree[2] (tile id slots). A B stage is reusable as soon as its MMA
// completed; the target norms the epilogue needs are fetched by each epilogue
// warp itself (cp.async, one chunk ahead) into its own double buffer.
constexpr int kExNCH = 128;
constexpr int kExEpiWarps = 8;
constexpr int kExThreads = (kExEpiWarps + 1) * 32;
constexpr int kExStages = 3;
constexpr int kExAcc = 2;

__host__ __device__ constexpr int dense_exact_min_blocks(int kmax) { return 1; }

template <int KMAX>
__global__ void __launch_bounds__(kExThreads, dense_exact_min_blocks(KMAX)) k_dense_exact(DenseArgs a) {
    extern __shared__ __align__(128) unsigned char smem[];
    if (!dense_exact_ok(a.lo_flag, a.dp)) return;  // the split-precision k_dense handles this join
    constexpr int NCH = kExNCH;
    const int KP = a.kp;
    const uint32_t sbo = (uint32_t)KP * 16u;
    const uint32_t a_bytes = (uint32_t)kDenseM * KP * 2, b_bytes = (uint32_t)NCH * KP * 2;
    unsigned char* sA = smem;
    unsigned char* sB = smem + a_bytes;  // [kExStages][b_bytes]
    __shared__ __align__(8) uint64_t bar_a, bar_full[kExStages], bar_sfree[kExStages], bar_mma[kExAcc],
        bar_afree[kExAcc], bar_tfull[2], bar_tfree[2];
    // target norms of a chunk, per epilogue warp (its 64 columns), double-buffered,
    // prefetched one chunk ahead by the warp itself with cp.async
    __shared__ __align__(16) float s_tnw[kExEpiWarps][2][kExNCH / 2];
    __shared__ uint32_t s_tmem;
    __shared__ int s_tile[2];
    __shared__ unsigned long long s_kth[2][kDenseM];  // {k-th d2 bits, tile seq} per half and row

    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    if (blockIdx.x == 0 && tid == 0) atomicMax(&a.counters->dense_terms, 1ull);
    if (warp == kExEpiWarps) tc::tmem_alloc(&s_tmem, (uint32_t)(kExAcc * NCH));
    if (tid == 0) {
        tc::mbar_init(smem_u32(&bar_a), 1);
        for (int i = 0; i < kExStages; ++i) {
            tc::mbar_init(smem_u32(&bar_full[i]), 1);
            tc::mbar_init(smem_u32(&bar_sfree[i]), 1);
        }
        for (int i = 0; i < kExAcc; ++i) {
            tc::mbar_init(smem_u32(&bar_mma[i]), 1);
            tc::mbar_init(smem_u32(&bar_afree[i]), kExEpiWarps);
        }
        for (int i = 0; i < 2; ++i) {
            tc::mbar_init(smem_u32(&bar_tfull[i]), 1);
            tc::mbar_init(smem_u32(&bar_tfree[i]), kExEpiWarps);
        }
        tc::mbar_fence_init();
    }
    for (int i = tid; i < 2 * kDenseM; i += blockDim.x) (&s_kth[0][0])[i] = ~0ull;
    fence_before();
    __syncthreads();
    fence_after();
    const uint32_t tmem = s_tmem;
    const int ntiles = *a.ntiles;

    if (warp == kExEpiWarps) {
        // ------------------------------------------------------- producer --
        if (lane == 0) {
            const uint32_t idesc = tc::idesc_bf16(kDenseM, NCH);
            uint32_t ph_a = 0;
            uint32_t g = 0;          // global chunk sequence (both roles count it identically)
            int last_acc = -1;
            uint32_t last_ph = 0;
            for (int t = 0;; ++t) {
                const int slot = t & 1;
                if (t >= 2) mbar_wait(smem_u32(&bar_tfree[slot]), ((t >> 1) - 1) & 1);
                const int tile = atomicAdd(a.counter, 1);
                *(volatile int*)&s_tile[slot] = tile;
                tc::mbar_arrive(smem_u32(&bar_tfull[slot]));
                if (tile >= ntiles) break;
                const int2 tl = a.tiles[tile];
                const int qc = tl.x;
                const size_t qp = (size_t)a.qoffp[qc] + tl.y;
                // the A tile is reloaded once every MMA of the previous tile is done
                if (last_acc >= 0) mbar_wait(smem_u32(&bar_mma[last_acc]), last_ph);
                expect_tx(smem_u32(&bar_a), a_bytes);
                bulk_g2s(smem_u32(sA), a.qhi + (qp >> 3) * sbo, a_bytes, smem_u32(&bar_a));
                ChunkIter<NCH> ld, mm;
                ld.start(a, qc);
                mm.start(a, qc);
                uint32_t lg = g;  // load cursor, runs up to kExStages chunks ahead of the MMA cursor
                auto issue_load = [&]() {
                    const int s = lg % kExStages;
                    if (lg >= (uint32_t)kExStages) mbar_wait(smem_u32(&bar_sfree[s]), ((lg / kExStages) - 1) & 1);
                    const uint32_t bar = smem_u32(&bar_full[s]);
                    expect_tx(bar, b_bytes);
                    const size_t p = (size_t)__ldg(a.toffp + ld.tc) + (size_t)ld.c * NCH;
                    bulk_g2s(smem_u32(sB + (size_t)s * b_bytes), a.thi + (p >> 3) * sbo, b_bytes, bar);
                    ++lg;
                    ld.advance(a);
                };
                bool a_ready = false;
                for (; mm.valid(); mm.advance(a), ++g) {
                    while (ld.valid() && lg < g + kExStages) issue_load();
                    if (!a_ready) {
                        mbar_wait(smem_u32(&bar_a), ph_a);
                        ph_a ^= 1u;
                        a_ready = true;
                    }
                    const int s = g % kExStages, c = g % kExAcc;
                    mbar_wait(smem_u32(&bar_full[s]), (g / kExStages) & 1);
                    if (g >= (uint32_t)kExAcc) mbar_wait(smem_u32(&bar_afree[c]), ((g / kExAcc) - 1) & 1);
                    fence_after();
                    const uint32_t aB = smem_u32(sA), bB = smem_u32(sB + (size_t)s * b_bytes);
                    const uint32_t d = tmem + (uint32_t)(c * NCH);
                    for (int ks = 0; ks < KP / 16; ++ks)
                        tc::mma_bf16(d, umma_desc(aB + ks * 256u, sbo), umma_desc(bB + ks * 256u, sbo), idesc, ks > 0);
                    tc::mma_commit(smem_u32(&bar_mma[c]));
                    tc::mma_commit(smem_u32(&bar_sfree[s]));
                    last_acc = c;
                    last_ph = (g / kExAcc) & 1;
                }
            }
        }
    } else {
        // ------------------------------------------------------- epilogue --
        const int quarter = warp & 3, half = warp >> 2;
        const int row = quarter * 32 + lane;
        // lanes 0-15 copy the warp's 64 norms of a chunk (16 B each) into buffer `sl`
        auto prefetch_tn = [&](const ChunkIter<NCH>& ci, int sl) {
            if (lane < 16) {
                const float* src = a.tn_raw + (size_t)__ldg(a.toffp + ci.tc) + (size_t)ci.c * NCH + half * (NCH / 2) + lane * 4;
                asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(smem_u32(&s_tnw[warp][sl][lane * 4])),
                             "l"(src)
                             : "memory");
            }
            asm volatile("cp.async.commit_group;" ::: "memory");
        };
        const uint32_t trow = tmem + ((uint32_t)(quarter * 32) << 16);
        const float INF = __int_as_float(0x7f800000);
        uint32_t g = 0;
        unsigned long long covered = 0;
        for (int t = 0;; ++t) {
            const int tslot = t & 1;
            mbar_wait(smem_u32(&bar_tfull[tslot]), (t >> 1) & 1);
            const int tile = *(volatile int*)&s_tile[tslot];
            __syncwarp();
            if (lane == 0) tc::mbar_arrive(smem_u32(&bar_tfree[tslot]));
            if (tile >= ntiles) break;
            const int2 tl = a.tiles[tile];
            const int qc = tl.x;
            const int qlo = a.qoff[qc], qsz = a.qoff[qc + 1] - qlo;
            const bool active = tl.y + row < qsz;
            const int qpos = qlo + tl.y + (active ? row : 0);
            const size_t qp = (size_t)a.qoffp[qc] + tl.y;
            const float na = active ? __ldg(a.qn + qp + row) : 0.f;
            RegTopK<KMAX> top;
            top.init(a.k);
            key_t kth = top.kth();
            const float ub = a.ub[qc];
            float kth2 = __fmul_ru(ub, ub);
            const unsigned long long tag = (unsigned long long)(unsigned)t;
            // the halves' k-th distances, exchanged with shared-memory atomics (a
            // reader may see the other's older value: any of them is a valid bound)
            unsigned long long* mine = &s_kth[half][row];
            unsigned long long* other = &s_kth[half ^ 1][row];
            atomicExch(mine, ((unsigned long long)__float_as_uint(kth2) << 32) | tag);
            ChunkIter<NCH> it;
            it.start(a, qc);
            int slot = 0;
            if (it.valid()) prefetch_tn(it, 0);
            for (; it.valid(); it.advance(a), ++g) {
                const int c = g % kExAcc;
                // (the epilogue must NOT wait on full[s]: that barrier may already be
                // one phase further -- the stage is refilled once the MMA is done)
                mbar_wait(smem_u32(&bar_mma[c]), (g / kExAcc) & 1);
                fence_after();
                const int nb = min(NCH, it.size - it.c * NCH);
                const int j0 = __ldg(a.toff + it.tc) + it.c * NCH;  // real (unpadded) first target
                // target norms ||b||^2 of this chunk's 64 columns (+inf on padding
                // rows): prefetch the next chunk's, then wait for this one's
                {
                    ChunkIter<NCH> nx = it;
                    const bool more = nx.advance(a);
                    if (more) prefetch_tn(nx, (slot ^ 1));
                    if (more) asm volatile("cp.async.wait_group 1;" ::: "memory");
                    else asm volatile("cp.async.wait_group 0;" ::: "memory");
                    __syncwarp();
                }
                const float* tn = s_tnw[warp][slot] - half * (NCH / 2);  // indexed by the chunk column
                float lim = kth2;
                const unsigned long long ot = atomicOr(other, 0ull);
                if ((ot & 0xffffffffull) == tag) lim = fminf(lim, __uint_as_float((uint32_t)(ot >> 32)));
                float thr = __fsub_ru(lim, na);  // keep t = ||b||^2 - 2 a.b iff t <= lim - ||a||^2
#pragma unroll 1
                for (int cb = 0; cb < NCH / 32; ++cb) {  // 16-column blocks of this half
                    const int col = half * (NCH / 2) + cb * 16;
                    if (col >= nb) break;  // warp-uniform
                    uint32_t v[16];
                    tc::tmem_ld16(trow + (uint32_t)(c * NCH + col), v);
                    float tt[16];
                    const float4* tn4 = reinterpret_cast<const float4*>(tn + col);
#pragma unroll
                    for (int j4 = 0; j4 < 4; ++j4) {
                        const float4 b4 = tn4[j4];
                        tt[4 * j4 + 0] = __fmaf_rn(-2.f, __uint_as_float(v[4 * j4 + 0]), b4.x);
                        tt[4 * j4 + 1] = __fmaf_rn(-2.f, __uint_as_float(v[4 * j4 + 1]), b4.y);
                        tt[4 * j4 + 2] = __fmaf_rn(-2.f, __uint_as_float(v[4 * j4 + 2]), b4.z);
                        tt[4 * j4 + 3] = __fmaf_rn(-2.f, __uint_as_float(v[4 * j4 + 3]), b4.w);
                    }
                    if (col + 16 > nb) {  // columns past the cluster's last target (next cluster's rows)
#pragma unroll
                        for (int j = 0; j < 16; ++j)
                            if (col + j >= nb) tt[j] = INF;
                    }
                    if (active && min_tree<16>(tt) <= thr) {  // 8 FMNMX3 (was 15 FMNMX)
                        unsigned m = 0;
#pragma unroll
                        for (int j = 0; j < 16; ++j) m |= (tt[j] <= thr ? 1u : 0u) << j;
                        while (m) {  // highest column first (members nearer the center)
                            const int j = 31 - __clz(m);
                            m &= ~(1u << j);
                            float tj = tt[0];
#pragma unroll
                            for (int u = 1; u < 16; ++u)
                                if (u == j) tj = tt[u];
                            const float d2 = tj + na;  // exact (integer < 2^24)
                            if (d2 <= kth2) {
                                const key_t key = make_key(d2, __ldg(a.torig + j0 + col + j));
                                if (key_lt(key, kth)) {
                                    top.insert(key);
                                    kth = top.kth();
                                    if (key_d2(kth) < kth2) {
                                        kth2 = key_d2(kth);
                                        thr = __fsub_ru(fminf(lim, kth2), na);
                                    }
                                }
                            }
                        }
                    }
                }
                fence_before();
                __syncwarp();  // (also: every lane is done with norm buffer `slot` before it is refilled)
                if (lane == 0) tc::mbar_arrive(smem_u32(&bar_afree[c]));  // accumulator c may be overwritten
                slot ^= 1;
                atomicExch(mine, ((unsigned long long)__float_as_uint(kth2) << 32) | tag);
                if (active && half == 0) covered += (unsigned long long)nb;
            }
            // merge the two halves' lists of each row (keys are distinct: disjoint columns)
            key_t* orow = a.topk_out + (int64_t)qpos * a.k;
            if (active && half == 1) {
#pragma unroll
                for (int q = 0; q < KMAX; ++q) {
                    const int r = q - (KMAX - a.k);
                    if (r >= 0) orow[r] = top.a[q];
                }
            }
            tc::bar_sync(1, kExEpiWarps * 32);
            if (active && half == 0) {
                for (int r = 0; r < a.k; ++r) {
                    const key_t key = orow[r];
                    if (key_lt(key, kth)) {
                        top.insert(key);
                        kth = top.kth();
                    }
                }
#pragma unroll
                for (int q = 0; q < KMAX; ++q) {
                    const int r = q - (KMAX - a.k);
                    if (r >= 0) orow[r] = top.a[q];
                }
            }
        }
        // counters: warps of half 0 only (all 32 lanes of a warp call add_counter)
        if (half == 0) add_counter(&a.counters->evals_dense, covered);
    }
    fence_before();
    __syncthreads();
    if (warp == kExEpiWarps) tc::tmem_dealloc(tmem, (uint32_t)(kExAcc * kExNCH));
}

template <int KMAX>
static sknn_status launch_dense_exact_k(Ctx& cx, const DenseArgs& a) {
    const size_t smem = (size_t)kDenseM * a.kp * 2 + kExStages * (size_t)kExNCH * a.kp * 2;
    SKNN_CUDA(cudaFuncSetAttribute(k_dense_exact<KMAX>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    int per_sm = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_dense_exact<KMAX>, kExThreads, smem);
    per_sm = std::max(1, std::min(per_sm, 512 / (kExAcc * kExNCH)));  // TMEM columns per SM
    k_dense_exact<KMAX><<<per_sm * cx.num_sms, kExThreads, smem, cx.stream>>>(a);
    cx.launched();
    return cx.check_launch("dense tiles (exact)");
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

// Both variants are launched; each reads the device-side exactness test
// (dense_exact_ok) and the one that does not apply exits at once, so the
// choice needs no host read-back (the join stays stream-ordered).
static sknn_status launch_dense_exact(Ctx& cx, const DenseArgs& a) {
    if (a.k <= 8) return launch_dense_exact_k<8>(cx, a);
    if (a.k <= 16) return launch_dense_exact_k<16>(cx, a);
    if (a.k <= 24) return launch_dense_exact_k<24>(cx, a);
    return launch_dense_exact_k<32>(cx, a);
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
                                int* lo_flag, int* amax_flag, DenseSide& out) {
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
                                        reinterpret_cast<__nv_bfloat16*>(out.lo), out.norm, out.norm_raw, lo_flag,
                                        amax_flag);
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
    // flags: [0] query lo part nonzero, [1] target lo part nonzero, [2] / [3]
    // max |x - o| (float bits) of the query / target side
    int* lo_flag;
    SKNN_TRY(cx.alloc_scratch((void**)&lo_flag, sizeof(int) * 4));
    SKNN_CUDA(cudaMemsetAsync(lo_flag, 0, sizeof(int) * 4, cx.stream));
    DenseSide tq, tt;
    SKNN_TRY(convert_side(cx, ts, kp, o, 1.f - eps_tc, true, lo_flag + 1, lo_flag + 3, tt));
    if (self) {
        tq = tt;
        tq.norm = tt.norm_raw;
        k_copy_flags<<<1, 32, 0, cx.stream>>>(lo_flag);
        cx.launched();
    } else {
        SKNN_TRY(convert_side(cx, qs, kp, o, 1.f, false, lo_flag, lo_flag + 2, tq));
    }
    DenseArgs a{};
    a.qrows = qs.rows; a.qoff = qs.off; a.qoffp = tq.offp; a.qhi = tq.hi; a.qlo = tq.lo; a.qn = tq.norm;
    a.trows = ts.rows; a.torig = ts.orig; a.toff = ts.off; a.toffp = tt.offp; a.thi = tt.hi; a.tlo = tt.lo;
    a.tn = tt.norm; a.tn_raw = tt.norm_raw; a.lo_flag = lo_flag;
    a.ub = l1.ub; a.dcand = l1.dcand; a.dcount = l1.dcount;
    a.tiles = l1.dtiles; a.ntiles = l1.dntiles; a.counter = l1.dntiles + 1;
    a.mt = ts.m; a.dp = ts.dp; a.kp = kp; a.k = p.k; a.eps_tc = eps_tc;
    a.topk_out = p.topk_out; a.counters = p.counters;
    if (!getenv("SKNN_DENSE_SPLIT_ONLY")) SKNN_TRY(launch_dense_exact(cx, a));  // ablation: split path only
    if (kp <= 64) return launch_dense_n<128>(cx, a);
    return launch_dense_n<64>(cx, a);
}

}  // namespace sknn
