// api.cu -- the C ABI (include/sknn.h): argument validation, the adaptive
// configuration (Fig. 8, §IV-D re-derived for B200), host/device staging,
// and the stage sequence of the Fig. 4 main procedure:
//   detLmNum -> init (build both sides) -> calUB + groupFilter -> pointFilter.
#include <cuda_runtime.h>
#include <math.h>
#include <stdint.h>
#include <string.h>

#include <algorithm>
#include <mutex>
#include <string>

#include "../../include/sknn.h"
#include "sknn_internal.cuh"
#include "sknn_launch.h"

namespace sknn {

static thread_local std::string g_last_error;
void set_last_error(const std::string& msg) { g_last_error = msg; }

static sknn_status fail(sknn_status st, const std::string& msg) {
    set_last_error(msg);
    return st;
}

// detLmNum: floor(3*sqrt(n)), clamped (reading R10)
static int det_lm_num(int64_t n, int32_t requested) {
    int64_t m = requested > 0 ? requested : (int64_t)floor(3.0 * sqrt((double)n));
    m = std::max<int64_t>(1, std::min<int64_t>(m, std::min<int64_t>(n, kMaxClusters)));
    return (int)m;
}

// R7: eta = (d + 8) * 2^-24
static float rounding_eta(int d) { return (float)((d + 8) * ldexp(1.0, -24)); }

struct DevInfo {
    int device = -1, num_sms = 0, max_threads_per_sm = 0, smem_per_sm = 0, regs_per_thread = 255, major = 0, minor = 0;
};

static sknn_status device_info(DevInfo& di) {
    int dev = 0;
    SKNN_CUDA(cudaGetDevice(&dev));
    static std::mutex mu;
    static DevInfo cache[64];
    std::lock_guard<std::mutex> lk(mu);
    if (dev >= 0 && dev < 64 && cache[dev].device == dev) {
        di = cache[dev];
        return SKNN_OK;
    }
    cudaDeviceProp p;
    SKNN_CUDA(cudaGetDeviceProperties(&p, dev));
    di.device = dev;
    di.num_sms = p.multiProcessorCount;
    di.max_threads_per_sm = p.maxThreadsPerMultiProcessor;
    di.smem_per_sm = (int)p.sharedMemPerMultiprocessor;
    di.major = p.major;
    di.minor = p.minor;
    if (di.major != 10 || di.minor != 0)
        return fail(SKNN_ERR_UNSUPPORTED, "device " + std::to_string(dev) + " is sm_" + std::to_string(p.major) +
                                              std::to_string(p.minor) + "; this library is built for sm_100a (B200)");
    if (!scratch_pool(dev)) return fail(SKNN_ERR_CUDA, "cudaMemPoolCreate failed");
    if (dev >= 0 && dev < 64) cache[dev] = di;
    return SKNN_OK;
}

// Private stream-ordered pool per device. Freed scratch stays reserved up to
// kPoolRetainBytes between calls (repeated joins reuse it without new
// cudaMalloc work); above that the driver releases it at synchronisation.
constexpr uint64_t kPoolRetainBytes = uint64_t(8) << 30;

cudaMemPool_t scratch_pool(int device) {
    static std::mutex mu;
    static cudaMemPool_t pools[64] = {};
    if (device < 0 || device >= 64) return nullptr;
    std::lock_guard<std::mutex> lk(mu);
    if (!pools[device]) {
        cudaMemPoolProps props;
        memset(&props, 0, sizeof(props));
        props.allocType = cudaMemAllocationTypePinned;
        props.location.type = cudaMemLocationTypeDevice;
        props.location.id = device;
        cudaMemPool_t p = nullptr;
        if (cudaMemPoolCreate(&p, &props) != cudaSuccess) {
            cudaGetLastError();
            return nullptr;
        }
        uint64_t thr = kPoolRetainBytes;
        cudaMemPoolSetAttribute(p, cudaMemPoolAttrReleaseThreshold, &thr);
        pools[device] = p;
    }
    return pools[device];
}

size_t usable_free_bytes(int device) {
    size_t free_b = 0, tot_b = 0;
    if (cudaMemGetInfo(&free_b, &tot_b) != cudaSuccess) {
        cudaGetLastError();
        return 0;
    }
    cudaMemPool_t p = scratch_pool(device);
    uint64_t reserved = 0, used = 0;
    if (p && cudaMemPoolGetAttribute(p, cudaMemPoolAttrReservedMemCurrent, &reserved) == cudaSuccess &&
        cudaMemPoolGetAttribute(p, cudaMemPoolAttrUsedMemCurrent, &used) == cudaSuccess && reserved > used)
        free_b += (size_t)(reserved - used);
    return free_b;
}

static sknn_options merge_options(const sknn_options* o) {
    sknn_options d;
    sknn_options_default(&d);
    if (!o) return d;
    size_t n = std::min(o->struct_size ? o->struct_size : sizeof(sknn_options), sizeof(sknn_options));
    memcpy(&d, o, n);
    d.struct_size = sizeof(sknn_options);
    if (d.landmark_trials <= 0) d.landmark_trials = 10;
    if (d.landmark_trials > 64) d.landmark_trials = 64;
    if (d.lloyd_iters < 0) d.lloyd_iters = 2;
    if (d.r_factor <= 0.f) d.r_factor = 0.25f;
    if (d.shard_count <= 1) { d.shard_count = 1; d.shard_rank = 0; }
    return d;
}

// Is the query array the index's build set (sknn_options.self_query)?
static bool index_self_query(const sknn_options& o, const void* Q, int64_t nq, const sknn_index* ix) {
    if (o.self_query < 0) return false;
    if (nq != ix->t.n) return false;
    if (o.self_query > 0) return true;
    return Q == ix->user_ptr;
}

enum PtrKind { PTR_DEVICE, PTR_HOST, PTR_BAD };

static PtrKind classify(const void* p, int dev) {
    cudaPointerAttributes at;
    cudaError_t e = cudaPointerGetAttributes(&at, p);
    if (e != cudaSuccess) {
        cudaGetLastError();
        return PTR_HOST;
    }
    if (at.type == cudaMemoryTypeDevice || at.type == cudaMemoryTypeManaged)
        return at.device == dev ? PTR_DEVICE : PTR_BAD;
    return PTR_HOST;
}

// Stage an input array on the device (copy when it is host memory).
static sknn_status stage_in(Ctx& cx, const void* p, size_t bytes, const void** out, bool* was_host) {
    PtrKind k = classify(p, cx.device);
    if (k == PTR_BAD) return fail(SKNN_ERR_NOT_DEVICE_PTR, "input pointer lives on another device");
    *was_host = (k == PTR_HOST);
    if (k == PTR_DEVICE) {
        *out = p;
        return SKNN_OK;
    }
    void* d;
    SKNN_TRY(cx.alloc_scratch(&d, bytes));
    SKNN_CUDA(cudaMemcpyAsync(d, p, bytes, cudaMemcpyHostToDevice, cx.stream));
    *out = d;
    return SKNN_OK;
}

static sknn_status stage_out(Ctx& cx, void* p, size_t bytes, void** dev, bool* was_host) {
    if (!p) {
        *dev = nullptr;
        *was_host = false;
        return SKNN_OK;
    }
    PtrKind k = classify(p, cx.device);
    if (k == PTR_BAD) return fail(SKNN_ERR_NOT_DEVICE_PTR, "output pointer lives on another device");
    *was_host = (k == PTR_HOST);
    if (k == PTR_DEVICE) {
        *dev = p;
        return SKNN_OK;
    }
    SKNN_TRY(cx.alloc_scratch(dev, bytes));
    return SKNN_OK;
}

struct Timer {
    bool on = false;
    cudaEvent_t ev[8] = {};
    int n = 0;
    cudaStream_t s = nullptr;
    void start(cudaStream_t st, bool enable) {
        on = enable;
        s = st;
        if (!on) return;
        for (int i = 0; i < 8; ++i) cudaEventCreate(&ev[i]);
        mark();
    }
    int mark() {
        if (!on) return -1;
        cudaEventRecord(ev[n], s);
        return n++;
    }
    float ms(int a, int b) const {
        if (!on || a < 0 || b < 0) return 0.f;
        float t = 0.f;
        cudaEventElapsedTime(&t, ev[a], ev[b]);
        return t;
    }
    ~Timer() {
        if (on)
            for (int i = 0; i < 8; ++i) cudaEventDestroy(ev[i]);
    }
};

static int choose_mapping(const sknn_options& o, const DevInfo& di, int64_t nq, int dp, int k) {
    if (o.mapping == SKNN_MAP_THREAD || o.mapping == SKNN_MAP_WARP || o.mapping == SKNN_MAP_BASIC) return o.mapping;
    if (k > 32) return scan_uses_bigk(k) ? SKNN_MAP_WARP : SKNN_MAP_THREAD;  // k_scan_bigk: warp per query
    // Fig. 8 bottom chooses query-level parallelism when
    // |Q| >= r*max_cur and several threads per query otherwise. Measured on
    // B200 (profiles/r01_sweep.md) the thread-per-query scan wins for every
    // dp <= 32 workload, even C1 (1,024 queries, formula: 64 threads/query),
    // because the sorted-member windows are short; the warp mapping is kept
    // for dp > 32, where a query no longer fits in one thread's registers.
    (void)di;
    (void)nq;
    return dp <= 32 ? SKNN_MAP_THREAD : SKNN_MAP_WARP;
}

static sknn_status validate(const float* Q, int64_t nq, const float* T, int64_t nt, int32_t d, int32_t k,
                            const float* out_dist) {
    if (!Q || !T || !out_dist) return fail(SKNN_ERR_INVALID_ARG, "Q, T and out_dist must be non-NULL");
    if (nq < 0) return fail(SKNN_ERR_INVALID_ARG, "nq < 0");
    if (nt <= 0) return fail(SKNN_ERR_INVALID_ARG, "nt <= 0");
    if (nt >= (int64_t(1) << 31) || nq >= (int64_t(1) << 31)) return fail(SKNN_ERR_INVALID_ARG, "nq, nt must be < 2^31");
    if (d <= 0) return fail(SKNN_ERR_INVALID_ARG, "d <= 0");
    if (k <= 0) return fail(SKNN_ERR_INVALID_ARG, "k <= 0");
    if ((int64_t)k > nt) return fail(SKNN_ERR_INVALID_ARG, "k > nt");
    if (k > SKNN_MAX_K) return fail(SKNN_ERR_UNSUPPORTED, "k > SKNN_MAX_K");
    return SKNN_OK;
}

struct Marks {
    int bt = -1, bq = -1, l1 = -1, dense = -1, scan = -1, end = -1;
};

// Elastic switch mode for level-1 (S8): 2 = every pair dense, 1 = none, 0 = cost model.
static int dense_mode_for(const sknn_options& o, int dp) {
    if (o.force_path == SKNN_PATH_DENSE) return 2;
    if (o.force_path == SKNN_PATH_SPARSE || o.force_path == SKNN_PATH_PARTIAL) return 1;
    // Measured per-pair cost ratio dense/sparse: ~0.3 at d = 16,
    // ~0.1 at d = 28, ~0.01 at d = 128. With the per-query bounds, the union
    // walk and the compile-time-k heap the sparse scan wins at every d <= 32
    // measured (C3 3.78 vs 3.95 ms, C3-int 6.74 vs 7.08 ms with the switch
    // armed), so the switch is armed only above dp = 32.
    if (o.dense_threshold > 0.f) return dense_supported(dp) ? 0 : 1;
    return (dp > 32 && dense_supported(dp)) ? 0 : 1;
}

// default window-share threshold of the elastic switch (dp > 16)
static float dense_tau_for(const sknn_options& o, int dp) {
    if (o.dense_threshold > 0.f) return o.dense_threshold;
    // measured with the exact-integer dense tiles (profiles/r02e_sweep_c4):
    // C4 tau 0.25 / 0.5 / 0.75 / all-dense = 62.4 / 67.6 / 103.3 / 193.9 ms
    return dp >= 64 ? 0.25f : 0.95f;
}

// The query half of Fig. 4 (lines 3-6) given both clustered sides:
// calUB + groupFilter (+ the elastic switch) -> dense tiles -> pointFilter.
static sknn_status query_core(Ctx& cx, const Side& qs, const Side& ts, int k, const sknn_options& o, int mapping,
                              int32_t* out_idx, float* out_dist, Counters* counters, Timer& tm, Marks& mk,
                              int* path_used) {
    const float eta = rounding_eta(ts.d);
    Level1 l1;
    Level1Params lp;
    lp.k = k;
    lp.eta = eta;
    lp.shard_rank = o.shard_count > 1 ? o.shard_rank : 0;
    lp.shard_count = o.shard_count > 1 ? o.shard_count : 1;
    // balanced query sharding: level-1 over every query cluster (replicated),
    // then the owner deal (run_shard_owner); the partial filter keeps interleave
    const bool balanced = lp.shard_count > 1 && o.shard_policy == 1 && o.force_path != SKNN_PATH_PARTIAL;
    const int shard_rank = lp.shard_rank, shard_count = lp.shard_count;
    if (balanced) {
        lp.shard_rank = 0;
        lp.shard_count = 1;
    }
    lp.dense_mode = dense_mode_for(o, ts.dp);
    lp.dense_tau = dense_tau_for(o, ts.dp);
    lp.ub_in = o.ub_in;
    if (lp.dense_mode == 2 && (!dense_supported(ts.dp) || k > 32)) {
        set_last_error("force_path = DENSE needs d <= 256 and k <= 32");
        return SKNN_ERR_UNSUPPORTED;
    }
    if (k > 32) lp.dense_mode = 1;  // the dense tiles keep a register top-k (k <= 32)
    const bool basic = mapping == SKNN_MAP_BASIC;
    if (basic) {
        if (k > 32 || o.force_path == SKNN_PATH_DENSE || o.force_path == SKNN_PATH_PARTIAL || shard_count > 1) {
            set_last_error("mapping = BASIC (ablation arm) runs the sparse full filter only, k <= 32, unsharded");
            return SKNN_ERR_UNSUPPORTED;
        }
        lp.dense_mode = 1;
    }
    DenseOrigin dorg;
    if (lp.dense_mode != 1) {
        SKNN_TRY(dense_prepare(cx, qs, ts, dorg));
        lp.dorg = &dorg;
    }
    if (lp.dense_mode == 0 && !lp.dorg) lp.dense_mode = 1;
    {
        NvtxRange r("sknn level-1 (calUB + groupFilter)");
        SKNN_TRY(run_level1(cx, qs, ts, lp, l1, counters));
    }
    if (balanced) SKNN_TRY(run_shard_owner(cx, qs, l1, shard_rank, shard_count));
    // Filter strength (§IV-D1, reading R13): the paper switches to the
    // partial level-2 filter when k/d > 8. Measured on B200 the
    // full filter wins every case once large k runs warp per query
    // (k_scan_bigk: C3 k = 512 15.0 ms full vs 61.0 ms partial; C2 k = 64,
    // k/d = 16: 4.5 vs 12.3 ms), so auto keeps the full filter and the partial
    // one runs on request (SKNN_PATH_PARTIAL).
    const bool partial = o.force_path == SKNN_PATH_PARTIAL;
    // the partial filter's passes take 32 queries per warp task (thread per query)
    const int tile = partial ? 32 : scan_tile_size(mapping, ts.dp, k);
    // Fig. 8: threads per query = nearest power of two of
    // r * max_cur / |Q| when |Q| < r * max_cur -- applied as the minimum split
    // of the thread-per-query scan's tiles (several warps per tile of queries)
    int fig8 = 1;
    {
        int dev = 0, sms = 148, mt_sm = 2048;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
        cudaDeviceGetAttribute(&mt_sm, cudaDevAttrMaxThreadsPerMultiProcessor, dev);
        const double rmax = (double)o.r_factor * sms * mt_sm;
        const int64_t nq_eff = qs.n / std::max(1, shard_count);
        if (nq_eff > 0 && (double)nq_eff < rmax) fig8 = 1 << (int)lround(log2(rmax / (double)nq_eff));
    }
    if (!basic)
        SKNN_TRY(run_tiles(cx, qs, tile, k, scan_resident_warps(cx, mapping, ts.dp, k), shard_rank, shard_count, l1,
                           fig8));
    mk.l1 = tm.mark();
    key_t* init_topk = nullptr;
    if (lp.dense_mode != 1) {
        SKNN_TRY(cx.alloc_scratch((void**)&init_topk, sizeof(key_t) * (size_t)qs.n * k));
        SKNN_TRY(run_dense_tiles(cx, qs, l1));
        DenseParams dpar;
        dpar.origin = dorg.o;
        dpar.k = k;
        dpar.eta = eta;
        dpar.topk_out = init_topk;
        dpar.counters = counters;
        NvtxRange r("sknn dense tiles");
        SKNN_TRY(run_dense(cx, qs, ts, l1, dpar));
        mk.dense = tm.mark();
    }
    ScanParams sp;
    sp.k = k;
    sp.eta = eta;
    sp.mapping = mapping;
    sp.out_squared = o.out_squared;
    sp.index_base = o.index_base;
    sp.out_idx = out_idx;
    sp.out_dist = out_dist;
    sp.counters = counters;
    sp.init_topk = init_topk;
    bool full = true;
    if (partial) {  // §IV-B1 partial level-2 filter
        bool fell_back = false;
        SKNN_TRY(run_partial(cx, qs, ts, l1, sp, &fell_back));
        full = fell_back;
        if (!fell_back) *path_used = SKNN_PATH_PARTIAL;
        // the full filter runs instead: its own task list (the partial passes'
        // 32-query split tasks are only valid for the thread-per-query scan)
        if (fell_back && scan_tile_size(mapping, ts.dp, k) != tile)
            SKNN_TRY(run_tiles(cx, qs, scan_tile_size(mapping, ts.dp, k), k,
                               scan_resident_warps(cx, mapping, ts.dp, k), shard_rank, shard_count, l1));
    }
    if (basic) {
        NvtxRange r("sknn level-2 scan (basic KNN-TI)");
        SKNN_TRY(run_scan_basic(cx, qs, ts, l1, sp));
    } else if (full) {
        NvtxRange r("sknn level-2 scan");
        SKNN_TRY(run_scan(cx, qs, ts, l1, sp));
    }
    mk.scan = tm.mark();
    return SKNN_OK;
}

static void fill_stats(sknn_stats* st, const Counters& c, int64_t nq, int64_t nt, const Timer& tm, const Marks& mk,
                       int mapping, int path, int mq, int mt, int launches) {
    size_t sz = st->struct_size ? std::min(st->struct_size, sizeof(sknn_stats)) : sizeof(sknn_stats);
    sknn_stats s;
    memset(&s, 0, sizeof(s));
    s.struct_size = sizeof(sknn_stats);
    s.pairs_total = (uint64_t)nq * (uint64_t)nt;
    s.dist_evals_sparse = c.evals_sparse;
    s.dist_evals_dense = c.evals_dense;
    s.dist_evals_brute = c.evals_brute;
    s.center_evals = c.center_evals;
    s.cand_pairs = c.cand_pairs;
    s.dense_pairs = c.dense_pairs;
    s.dist_recompute = c.dist_recompute;
    s.topk_inserts = c.topk_inserts;
    s.rows_loaded = c.rows_loaded;
    s.dense_terms = (uint32_t)c.dense_terms;
    s.ms_total = tm.ms(0, mk.end);
    s.ms_build_t = tm.ms(0, mk.bt);
    s.ms_build_q = mk.bq >= 0 ? tm.ms(mk.bt, mk.bq) : 0.f;
    const int prev = mk.bq >= 0 ? mk.bq : mk.bt;
    s.ms_level1 = mk.l1 >= 0 ? tm.ms(prev, mk.l1) : 0.f;
    s.ms_dense = mk.dense >= 0 ? tm.ms(mk.l1, mk.dense) : 0.f;
    s.ms_sparse = mk.scan >= 0 ? tm.ms(mk.dense >= 0 ? mk.dense : mk.l1, mk.scan) : 0.f;
    s.ms_final = 0.f;
    s.mapping_used = mapping;
    s.path_used = (path == SKNN_PATH_BRUTE || path == SKNN_PATH_PARTIAL) ? path
                                                                         : (c.dense_pairs ? SKNN_PATH_DENSE : SKNN_PATH_SPARSE);
    s.mq = mq;
    s.mt = mt;
    s.kernel_launches = launches;
    memcpy(st, &s, sz);
}

// Private non-blocking stream per device for the forked query-side build.
static cudaStream_t side_stream(int dev) {
    static std::mutex mu;
    static cudaStream_t s[64] = {};
    if (dev < 0 || dev >= 64) return nullptr;
    std::lock_guard<std::mutex> lk(mu);
    if (!s[dev] && cudaStreamCreateWithFlags(&s[dev], cudaStreamNonBlocking) != cudaSuccess) {
        cudaGetLastError();
        s[dev] = nullptr;
    }
    return s[dev];
}

// Shared body of sknn_join_ex / sknn_query.
static sknn_status run_join(const float* Q, int64_t nq, const float* T, int64_t nt, int32_t d, int32_t k,
                            int32_t* out_idx, float* out_dist, const sknn_options* opt_in, sknn_stats* stats,
                            cudaStream_t stream, const sknn_index* index, bool capturing = false,
                            const sknn_index* qindex = nullptr, bool defer_sync = false) {
    NvtxRange nvtx_call(qindex ? "sknn_join_indexed" : (index ? "sknn_query" : "sknn_join"));
    // a query index supplies the clustered query side (Q is not read)
    static const float kNoQ = 0.f;
    if (qindex) Q = &kNoQ;
    SKNN_TRY(validate(Q, nq, T ? T : Q, nt, d, k, out_dist));
    if (nq == 0) {
        if (stats) {
            memset(stats, 0, sizeof(sknn_stats));
            stats->struct_size = sizeof(sknn_stats);
        }
        return SKNN_OK;
    }
    DevInfo di;
    SKNN_TRY(device_info(di));
    if (index && index->device != di.device) return fail(SKNN_ERR_WRONG_DEVICE, "index built on another device");
    sknn_options o = merge_options(opt_in ? opt_in : (index ? &index->opt : nullptr));
    if (opt_in && index) {  // clustering of the index side is fixed; query-side knobs come from opt_in
        o.n_clusters_t = index->t.m;
    }
    Ctx cx;
    cx.stream = stream;
    cx.device = di.device;
    cx.num_sms = di.num_sms;
    cx.capturing = capturing;
    Timer tm;
    tm.start(stream, stats != nullptr);
    sknn_status st = SKNN_OK;
    const int dp = (d + 3) & ~3;
    const bool self = qindex ? qindex == index : (index ? index_self_query(o, Q, nq, index) : (Q == T && nq == nt));
    int mapping = choose_mapping(o, di, nq, dp, k);
    // dense-only (every pair, k_brute_tiled): forced, or auto at high d, where
    // the TI filters keep most pairs and the scans' per-lane rows cost more
    // than a tiled contraction (measured: arcene/dorothea shapes)
    const bool dense_only = o.force_path == SKNN_PATH_BRUTE ||
                            (o.force_path == SKNN_PATH_AUTO && dp >= kDenseOnlyDp && k <= 32 && !qindex &&
                             o.shard_count <= 1 && !o.ub_in && o.mapping != SKNN_MAP_BASIC);
    int path = dense_only ? SKNN_PATH_BRUTE : SKNN_PATH_SPARSE;
    Marks mk;
    int mq = 0, mt = 0;
    Counters host_c;
    memset(&host_c, 0, sizeof(host_c));
    bool q_host = false, t_host = false, oi_host = false, od_host = false;
    const float* dQ = nullptr;
    const float* dT = nullptr;
    int32_t* d_oidx = nullptr;
    float* d_odist = nullptr;
    Counters* counters = nullptr;
    Ctx cq;  // forked query-side build (Q != T joins)
    cudaEvent_t ev_fork = nullptr, ev_join = nullptr;
    // Q != T join with a forked query-side build: Q is staged on the forked
    // stream after T's copy, so (host buffers) its host->device copy overlaps
    // the target-side build instead of preceding it
    const bool fork_q = !index && !self && !qindex && path != SKNN_PATH_BRUTE;
    do {
        const void* tmp;
        if (!qindex && !fork_q) {
            if ((st = stage_in(cx, Q, sizeof(float) * nq * d, &tmp, &q_host)) != SKNN_OK) break;
            dQ = (const float*)tmp;
        }
        if (!index) {
            if (self) {
                dT = dQ;
            } else {
                if ((st = stage_in(cx, T, sizeof(float) * nt * d, &tmp, &t_host)) != SKNN_OK) break;
                dT = (const float*)tmp;
            }
        }
        void* vo;
        if ((st = stage_out(cx, out_idx, sizeof(int32_t) * nq * k, &vo, &oi_host)) != SKNN_OK) break;
        d_oidx = (int32_t*)vo;
        if ((st = stage_out(cx, out_dist, sizeof(float) * nq * k, &vo, &od_host)) != SKNN_OK) break;
        d_odist = (float*)vo;
        if ((st = cx.alloc_scratch((void**)&counters, sizeof(Counters))) != SKNN_OK) break;
        if (cudaMemsetAsync(counters, 0, sizeof(Counters), stream) != cudaSuccess) {
            st = fail(SKNN_ERR_CUDA, "cudaMemsetAsync(counters) failed");
            break;
        }
        if (path == SKNN_PATH_BRUTE) {
            if (qindex) {
                st = fail(SKNN_ERR_INVALID_ARG, "force_path = BRUTE is not available for sknn_join_indexed");
                break;
            }
            ScanParams sp;
            sp.k = k;
            sp.out_squared = o.out_squared;
            sp.index_base = o.index_base;
            sp.out_idx = d_oidx;
            sp.out_dist = d_odist;
            sp.counters = counters;
            if (k > 32) {
                st = fail(SKNN_ERR_UNSUPPORTED, "force_path = BRUTE supports k <= 32");
                break;
            }
            const char* eb = getenv("SKNN_BRUTE");  // "warp": the warp-per-query anchor kernel (caller rows only)
            if (eb && !strcmp(eb, "warp") && !index) {
                mapping = SKNN_MAP_WARP;
                st = run_brute(cx, dQ, nq, dT, nt, d, sp);
            } else {
                mapping = SKNN_MAP_THREAD;
                // an index holds its rows permuted and padded to dp, with the original ids
                st = index ? run_brute_tiled(cx, dQ, nq, d, index->t.rows, nt, index->t.dp, index->t.orig, d, sp)
                           : run_brute_tiled(cx, dQ, nq, d, dT, nt, d, nullptr, d, sp);
            }
            mk.bt = tm.mark();
            mk.scan = mk.bt;
            break;
        }
        Side ts_local, qs_local;
        const Side* ts;
        // A Q != T join clusters both sides: the query side is built on a forked
        // stream concurrently with the target side (both are chains of mostly
        // small, latency-bound kernels; the joins and frees stay stream-ordered,
        // and a graph capture follows the fork/join events)
        if (fork_q) {
            cq.stream = side_stream(di.device);
            cq.device = cx.device;
            cq.num_sms = cx.num_sms;
            cq.capturing = capturing;
            if (!cq.stream || cudaEventCreateWithFlags(&ev_fork, cudaEventDisableTiming) != cudaSuccess ||
                cudaEventCreateWithFlags(&ev_join, cudaEventDisableTiming) != cudaSuccess ||
                cudaEventRecord(ev_fork, stream) != cudaSuccess || cudaStreamWaitEvent(cq.stream, ev_fork, 0) != cudaSuccess) {
                st = fail(SKNN_ERR_CUDA, "fork of the query-side build failed");
                break;
            }
            if ((st = stage_in(cq, Q, sizeof(float) * nq * d, &tmp, &q_host)) != SKNN_OK) break;
            dQ = (const float*)tmp;
            int m = det_lm_num(nq, o.n_clusters_q);
            NvtxRange r("sknn build query side (forked stream)");
            if ((st = build_side(cq, dQ, nq, d, m, o.landmark_trials, o.lloyd_iters, o.seed ^ 0x51ull, qs_local)) !=
                SKNN_OK)
                break;
            cq.free_scratch();
            if (cudaEventRecord(ev_join, cq.stream) != cudaSuccess) {
                st = fail(SKNN_ERR_CUDA, "join of the query-side build failed");
                break;
            }
        }
        if (index) {
            ts = &index->t;
        } else {
            int m = det_lm_num(nt, o.n_clusters_t);
            NvtxRange r("sknn build target side");
            if ((st = build_side(cx, dT, nt, d, m, o.landmark_trials, o.lloyd_iters, o.seed, ts_local)) != SKNN_OK)
                break;
            ts = &ts_local;
        }
        mk.bt = tm.mark();
        const Side* qs;
        if (self) {
            qs = ts;
        } else if (qindex) {
            qs = &qindex->t;
        } else if (!fork_q) {  // query of a resident index: cluster Q here
            int m = det_lm_num(nq, o.n_clusters_q);
            NvtxRange r("sknn build query side");
            if ((st = build_side(cx, dQ, nq, d, m, o.landmark_trials, o.lloyd_iters, o.seed ^ 0x51ull, qs_local)) !=
                SKNN_OK)
                break;
            qs = &qs_local;
            mk.bq = tm.mark();
        } else {
            if (cudaStreamWaitEvent(stream, ev_join, 0) != cudaSuccess) {
                st = fail(SKNN_ERR_CUDA, "join of the query-side build failed");
                break;
            }
            // the query side's arrays are used (and freed) on `stream` from here on
            cx.persistent.insert(cx.persistent.end(), cq.persistent.begin(), cq.persistent.end());
            cq.persistent.clear();
            cx.launches += cq.launches;
            cudaEventDestroy(ev_fork);
            cudaEventDestroy(ev_join);
            ev_fork = ev_join = nullptr;
            qs = &qs_local;
            mk.bq = tm.mark();
        }
        mq = qs->m;
        mt = ts->m;
        st = query_core(cx, *qs, *ts, k, o, mapping, d_oidx, d_odist, counters, tm, mk, &path);
    } while (0);
    if (st == SKNN_OK) {
        if (oi_host) {
            cudaError_t e = cudaMemcpyAsync(out_idx, d_oidx, sizeof(int32_t) * nq * k, cudaMemcpyDeviceToHost, stream);
            if (e != cudaSuccess) st = fail(SKNN_ERR_CUDA, std::string("D2H out_idx: ") + cudaGetErrorString(e));
        }
        if (od_host) {
            cudaError_t e = cudaMemcpyAsync(out_dist, d_odist, sizeof(float) * nq * k, cudaMemcpyDeviceToHost, stream);
            if (e != cudaSuccess) st = fail(SKNN_ERR_CUDA, std::string("D2H out_dist: ") + cudaGetErrorString(e));
        }
        if (stats && counters) cudaMemcpyAsync(&host_c, counters, sizeof(Counters), cudaMemcpyDeviceToHost, stream);
        mk.end = tm.mark();
    }
    if (ev_fork) {  // an error left the forked build unjoined: join it, free its memory
        if (!ev_join || cudaEventRecord(ev_join, cq.stream) != cudaSuccess) cudaStreamSynchronize(cq.stream);
        else cudaStreamWaitEvent(stream, ev_join, 0);
        cq.free_all();
        cudaEventDestroy(ev_fork);
        if (ev_join) cudaEventDestroy(ev_join);
    }
    int launches = cx.launches;
    cx.free_all();
    // host buffers are synchronised before returning, unless the caller (the
    // overlapped out-of-core batches) passed pinned buffers and syncs itself
    if (st == SKNN_OK && (stats || ((oi_host || od_host || q_host || t_host) && !defer_sync))) {
        cudaError_t e = cudaStreamSynchronize(stream);
        if (e != cudaSuccess) st = fail(SKNN_ERR_CUDA, std::string("kernel execution failed: ") + cudaGetErrorString(e));
    }
    if (st == SKNN_OK && stats)
        fill_stats(stats, host_c, nq, nt, tm, mk, mapping, path, mq, mt, launches);
    return st;
}

// ------------------------------------------------------------ CUDA graphs --
// A whole join is ~25-30 stream-ordered launches with no host round trip, so
// on small (launch-bound) joins the launch gaps are a visible share of the
// step. A join whose key (device, pointers, sizes, options) was seen before is
// recorded ONCE into a CUDA graph (stream capture on a private stream; scratch
// allocations become graph memory nodes) and replayed with one cudaGraphLaunch
// afterwards. The graph reads the arrays at the recorded addresses, so a replay
// on new contents of the same buffers computes the join of the new contents.
// Only device-pointer calls without stats, outside the partial filter (which
// sizes its buffer on the host), with a modest scratch footprint.
struct GraphKey {
    int device;
    const void *Q, *T, *oi, *od;
    int64_t nq, nt;
    int32_t d, k;
    sknn_options o;
    bool operator==(const GraphKey& b) const {
        return device == b.device && Q == b.Q && T == b.T && oi == b.oi && od == b.od && nq == b.nq && nt == b.nt &&
               d == b.d && k == b.k && memcmp(&o, &b.o, sizeof(o)) == 0;
    }
};
struct GraphEntry {
    GraphKey key;
    cudaGraphExec_t exec = nullptr;  // nullptr: seen once, not yet recorded
    uint64_t used = 0;
};
constexpr int kGraphCache = 8;
static std::mutex g_graph_mu;
static GraphEntry g_graphs[kGraphCache];
static int g_graph_n = 0;
static uint64_t g_graph_clock = 0;

static cudaStream_t capture_stream(int dev) {
    static cudaStream_t s[64] = {};
    if (dev < 0 || dev >= 64) return nullptr;
    if (!s[dev] && cudaStreamCreateWithFlags(&s[dev], cudaStreamNonBlocking) != cudaSuccess) {
        cudaGetLastError();
        s[dev] = nullptr;
    }
    return s[dev];
}

static sknn_status run_join_graphed(const float* Q, int64_t nq, const float* T, int64_t nt, int32_t d, int32_t k,
                                    int32_t* out_idx, float* out_dist, const sknn_options* opt, sknn_stats* stats,
                                    cudaStream_t stream) {
    auto eager = [&]() { return run_join(Q, nq, T, nt, d, k, out_idx, out_dist, opt, stats, stream, nullptr); };
    if (stats || !Q || !T || !out_dist || nq <= 0 || nt <= 0 || d <= 0 || k <= 0) return eager();
    const sknn_options o = merge_options(opt);
    if (o.use_graph < 0 || o.force_path == SKNN_PATH_PARTIAL) return eager();
    DevInfo di;
    if (device_info(di) != SKNN_OK) return eager();
    if (classify(Q, di.device) != PTR_DEVICE || classify(T, di.device) != PTR_DEVICE ||
        classify(out_dist, di.device) != PTR_DEVICE || (out_idx && classify(out_idx, di.device) != PTR_DEVICE))
        return eager();
    const int dp = (d + 3) & ~3;
    const double footprint = (double)(nq + nt) * (4.0 * dp + 8.0 * k + 64.0);
    if (footprint > (double)(1u << 30)) return eager();  // large joins are not launch-bound
    GraphKey key;
    memset(&key, 0, sizeof(key));
    key.device = di.device; key.Q = Q; key.T = T; key.oi = out_idx; key.od = out_dist;
    key.nq = nq; key.nt = nt; key.d = d; key.k = k; key.o = o;
    std::lock_guard<std::mutex> lk(g_graph_mu);
    int slot = -1;
    for (int i = 0; i < g_graph_n; ++i)
        if (g_graphs[i].key == key) slot = i;
    if (slot >= 0 && g_graphs[slot].exec) {
        g_graphs[slot].used = ++g_graph_clock;
        SKNN_CUDA(cudaGraphLaunch(g_graphs[slot].exec, stream));
        return SKNN_OK;
    }
    if (slot < 0) {  // first sighting: run eagerly, remember the key
        if (g_graph_n < kGraphCache) {
            slot = g_graph_n++;
        } else {
            slot = 0;
            for (int i = 1; i < kGraphCache; ++i)
                if (g_graphs[i].used < g_graphs[slot].used) slot = i;
            if (g_graphs[slot].exec) cudaGraphExecDestroy(g_graphs[slot].exec);
        }
        g_graphs[slot].key = key;
        g_graphs[slot].exec = nullptr;
        g_graphs[slot].used = ++g_graph_clock;
        return eager();
    }
    // second sighting: record the join once, then launch the graph
    cudaStream_t cap = capture_stream(di.device);
    if (!cap) return eager();
    if (cudaStreamBeginCapture(cap, cudaStreamCaptureModeThreadLocal) != cudaSuccess) {
        cudaGetLastError();
        return eager();
    }
    sknn_status st = run_join(Q, nq, T, nt, d, k, out_idx, out_dist, opt, nullptr, cap, nullptr, true);
    cudaGraph_t g = nullptr;
    cudaError_t e = cudaStreamEndCapture(cap, &g);
    cudaGraphExec_t exec = nullptr;
    if (st == SKNN_OK && e == cudaSuccess && g) e = cudaGraphInstantiate(&exec, g, 0);
    if (g) cudaGraphDestroy(g);
    if (st != SKNN_OK || e != cudaSuccess || !exec) {
        cudaGetLastError();
        g_graphs[slot].used = ++g_graph_clock;  // stays "seen": try to record again next time
        return eager();
    }
    g_graphs[slot].exec = exec;
    g_graphs[slot].used = ++g_graph_clock;
    SKNN_CUDA(cudaGraphLaunch(exec, stream));
    return SKNN_OK;
}

}  // namespace sknn

using namespace sknn;

extern "C" {

void sknn_options_default(sknn_options* o) {
    if (!o) return;
    memset(o, 0, sizeof(*o));
    o->struct_size = sizeof(sknn_options);
    o->landmark_trials = 10;
    o->lloyd_iters = 2;
    o->seed = 0x5eedull;
    o->force_path = SKNN_PATH_AUTO;
    o->mapping = SKNN_MAP_AUTO;
    o->r_factor = 0.25f;
}

sknn_status sknn_join(const float* Q, int64_t nq, const float* T, int64_t nt, int32_t d, int32_t k, int32_t* out_idx,
                      float* out_dist, sknn_stream_t stream) {
    return run_join_graphed(Q, nq, T, nt, d, k, out_idx, out_dist, nullptr, nullptr, (cudaStream_t)stream);
}

sknn_status sknn_join_ex(const float* Q, int64_t nq, const float* T, int64_t nt, int32_t d, int32_t k,
                         int32_t* out_idx, float* out_dist, const sknn_options* opt, sknn_stats* stats,
                         sknn_stream_t stream) {
    return run_join_graphed(Q, nq, T, nt, d, k, out_idx, out_dist, opt, stats, (cudaStream_t)stream);
}

static sknn_status build_index_impl(const float* T, int64_t nt, int32_t d, const sknn_options* opt, sknn_index** out,
                                    sknn_stream_t stream_, const BuildShard* shard);

sknn_status sknn_build(const float* T, int64_t nt, int32_t d, const sknn_options* opt, sknn_index** out,
                       sknn_stream_t stream_) {
    return build_index_impl(T, nt, d, opt, out, stream_, nullptr);
}

int32_t sknn_cluster_count(int64_t n, const sknn_options* opt) {
    const sknn_options o = merge_options(opt);
    return n > 0 ? det_lm_num(n, o.n_clusters_t) : 0;
}

sknn_status sknn_build_from_assignment(const float* T, int64_t nt, int32_t d, const sknn_options* opt,
                                       const float* centers, int32_t m, const int32_t* cid, const float* dist,
                                       sknn_index** out, sknn_stream_t stream) {
    if (!centers || !cid || !dist) return fail(SKNN_ERR_INVALID_ARG, "NULL pointer");
    if (m != sknn_cluster_count(nt, opt)) return fail(SKNN_ERR_INVALID_ARG, "m differs from sknn_cluster_count");
    DevInfo di;
    SKNN_TRY(device_info(di));
    if (classify(centers, di.device) != PTR_DEVICE || classify(cid, di.device) != PTR_DEVICE ||
        classify(dist, di.device) != PTR_DEVICE)
        return fail(SKNN_ERR_NOT_DEVICE_PTR, "centers, cid and dist must be device memory");
    BuildShard sh;
    sh.mode = 2;
    sh.centers_in = centers;
    sh.cid_in = cid;
    sh.dist_in = dist;
    return build_index_impl(T, nt, d, opt, out, stream, &sh);
}

sknn_status sknn_build_assign_shard(const float* T, int64_t nt, int32_t d, const sknn_options* opt, int64_t row_lo,
                                    int64_t row_hi, float* centers_out, int32_t* cid_out, float* dist_out,
                                    sknn_stream_t stream) {
    if (!centers_out || !cid_out || !dist_out) return fail(SKNN_ERR_INVALID_ARG, "NULL pointer");
    if (row_lo < 0 || row_hi < row_lo || row_hi > nt || (row_lo % 8) != 0)
        return fail(SKNN_ERR_INVALID_ARG, "rows must satisfy 0 <= row_lo <= row_hi <= nt, row_lo % 8 == 0");
    DevInfo di;
    SKNN_TRY(device_info(di));
    if (classify(centers_out, di.device) != PTR_DEVICE || classify(cid_out, di.device) != PTR_DEVICE ||
        classify(dist_out, di.device) != PTR_DEVICE)
        return fail(SKNN_ERR_NOT_DEVICE_PTR, "outputs must be device memory");
    BuildShard sh;
    sh.mode = 1;
    sh.lo = row_lo;
    sh.hi = row_hi;
    sh.centers_out = centers_out;
    sh.cid_out = cid_out;
    sh.dist_out = dist_out;
    sknn_index* tmp = nullptr;
    sknn_status st = build_index_impl(T, nt, d, opt, &tmp, stream, &sh);
    if (tmp) sknn_index_free(tmp);  // the partial side is not an index
    return st;
}

static sknn_status build_index_impl(const float* T, int64_t nt, int32_t d, const sknn_options* opt, sknn_index** out,
                                    sknn_stream_t stream_, const BuildShard* shard) {
    if (!out) return fail(SKNN_ERR_INVALID_ARG, "out is NULL");
    *out = nullptr;
    if (!T) return fail(SKNN_ERR_INVALID_ARG, "T is NULL");
    if (nt <= 0 || nt >= (int64_t(1) << 31)) return fail(SKNN_ERR_INVALID_ARG, "nt must be in [1, 2^31)");
    if (d <= 0) return fail(SKNN_ERR_INVALID_ARG, "d <= 0");
    DevInfo di;
    SKNN_TRY(device_info(di));
    cudaStream_t stream = (cudaStream_t)stream_;
    sknn_options o = merge_options(opt);
    Ctx cx;
    cx.stream = stream;
    cx.device = di.device;
    cx.num_sms = di.num_sms;
    sknn_index* ix = new (std::nothrow) sknn_index();
    if (!ix) return fail(SKNN_ERR_OOM, "host allocation of the index failed");
    ix->device = di.device;
    ix->user_ptr = T;
    ix->opt = o;
    sknn_status st;
    do {
        const void* dT;
        bool th;
        if ((st = stage_in(cx, T, sizeof(float) * nt * d, &dT, &th)) != SKNN_OK) break;
        int m = det_lm_num(nt, o.n_clusters_t);
        st = build_side(cx, (const float*)dT, nt, d, m, o.landmark_trials, o.lloyd_iters, o.seed, ix->t, shard);
    } while (0);
    cx.free_scratch();
    if (st == SKNN_OK) {
        cudaError_t e = cudaStreamSynchronize(stream);  // the index is usable on any stream afterwards
        if (e != cudaSuccess) st = fail(SKNN_ERR_CUDA, std::string("index build failed: ") + cudaGetErrorString(e));
    }
    if (st != SKNN_OK) {
        cx.free_all();
        delete ix;
        return st;
    }
    *out = ix;
    return SKNN_OK;
}

// Out-of-core batches, overlapped (NEXT-4): batch b runs on stream s[b % 2]
// (the caller's stream and one private stream), so batch b's host->device
// copy and kernels overlap batch b-1's device->host copy. Host buffers the
// caller did not page-lock go through page-locked staging buffers (a
// cudaMemcpyAsync into pageable memory blocks the host thread until it
// completes, which would serialise the batches): rows are staged on the host
// while the device runs the previous batch, and a batch's results are copied
// out of staging once its completion event fires. Every batch is the same
// exact query, so the rows equal one unbatched call.
static bool pinned_host(const void* p) {
    cudaPointerAttributes at;
    if (cudaPointerGetAttributes(&at, p) != cudaSuccess) {
        cudaGetLastError();
        return false;
    }
    return at.type == cudaMemoryTypeHost;
}

static sknn_status query_batches_overlapped(const sknn_index* index, const float* Q, int64_t nq, int32_t k,
                                            int32_t* out_idx, float* out_dist, const sknn_options* opt, int64_t B,
                                            cudaStream_t user) {
    const int d = index->t.d;
    const bool q_pin = pinned_host(Q), oi_pin = !out_idx || pinned_host(out_idx), od_pin = pinned_host(out_dist);
    if (!(q_pin && oi_pin && od_pin)) {  // staging: at most 256 MB of rows per slot (SKNN_OOC_STAGE=1 only)
        const int64_t row = 4ll * d + 8ll * k;
        B = std::max<int64_t>(k, std::min<int64_t>(B, (256ll << 20) / row));
    }
    cudaStream_t s[2] = {user, nullptr};
    cudaEvent_t done[2] = {nullptr, nullptr}, start = nullptr;
    float* sq[2] = {nullptr, nullptr};
    int32_t* si[2] = {nullptr, nullptr};
    float* sd[2] = {nullptr, nullptr};
    int64_t pend_b0[2] = {-1, -1}, pend_nb[2] = {0, 0};
    sknn_status st = SKNN_OK;
    auto cuda_ok = [&](cudaError_t e, const char* what) {
        if (e == cudaSuccess) return true;
        st = fail(SKNN_ERR_CUDA, std::string(what) + ": " + cudaGetErrorString(e));
        return false;
    };
    // results of the batch in `slot` (already complete) into the caller's buffers
    auto finish = [&](int slot) {
        if (pend_b0[slot] < 0) return;
        if (!cuda_ok(cudaEventSynchronize(done[slot]), "batch")) return;
        const int64_t b0 = pend_b0[slot], nb = pend_nb[slot];
        if (!od_pin) memcpy(out_dist + b0 * k, sd[slot], sizeof(float) * nb * k);
        if (!oi_pin) memcpy(out_idx + b0 * k, si[slot], sizeof(int32_t) * nb * k);
        pend_b0[slot] = -1;
    };
    do {
        if (!cuda_ok(cudaStreamCreateWithFlags(&s[1], cudaStreamNonBlocking), "stream")) break;
        if (!cuda_ok(cudaEventCreateWithFlags(&start, cudaEventDisableTiming), "event")) break;
        if (!cuda_ok(cudaEventCreateWithFlags(&done[0], cudaEventDisableTiming), "event")) break;
        if (!cuda_ok(cudaEventCreateWithFlags(&done[1], cudaEventDisableTiming), "event")) break;
        // the private stream starts after the work the caller queued before the call
        if (!cuda_ok(cudaEventRecord(start, user), "event")) break;
        if (!cuda_ok(cudaStreamWaitEvent(s[1], start, 0), "event")) break;
        for (int i = 0; i < 2 && st == SKNN_OK; ++i) {
            if (!q_pin) cuda_ok(cudaHostAlloc((void**)&sq[i], sizeof(float) * B * d, cudaHostAllocDefault), "staging");
            if (!oi_pin && st == SKNN_OK)
                cuda_ok(cudaHostAlloc((void**)&si[i], sizeof(int32_t) * B * k, cudaHostAllocDefault), "staging");
            if (!od_pin && st == SKNN_OK)
                cuda_ok(cudaHostAlloc((void**)&sd[i], sizeof(float) * B * k, cudaHostAllocDefault), "staging");
        }
        if (st != SKNN_OK) break;
        int b = 0;
        for (int64_t b0 = 0; b0 < nq && st == SKNN_OK; b0 += B, ++b) {
            const int slot = b & 1;
            const int64_t nb = std::min(B, nq - b0);
            finish(slot);  // batch b-2: its staging buffers are free again
            if (st != SKNN_OK) break;
            const float* qb = Q + b0 * d;
            if (!q_pin) {
                memcpy(sq[slot], qb, sizeof(float) * nb * d);
                qb = sq[slot];
            }
            int32_t* ob = out_idx ? (oi_pin ? out_idx + b0 * k : si[slot]) : nullptr;
            float* db = od_pin ? out_dist + b0 * k : sd[slot];
            st = run_join(qb, nb, nullptr, index->t.n, d, k, ob, db, opt, nullptr, s[slot], index, false, nullptr,
                          /*defer_sync=*/true);
            if (st != SKNN_OK) break;
            if (!cuda_ok(cudaEventRecord(done[slot], s[slot]), "event")) break;
            pend_b0[slot] = b0;
            pend_nb[slot] = nb;
        }
        // oldest first
        const int last = (b - 1) & 1;
        finish(last ^ 1);
        finish(last);
    } while (0);
    if (s[1]) {
        cudaStreamSynchronize(s[1]);
        cudaStreamDestroy(s[1]);
    }
    cudaStreamSynchronize(user);
    for (int i = 0; i < 2; ++i) {
        if (sq[i]) cudaFreeHost(sq[i]);
        if (si[i]) cudaFreeHost(si[i]);
        if (sd[i]) cudaFreeHost(sd[i]);
        if (done[i]) cudaEventDestroy(done[i]);
    }
    if (start) cudaEventDestroy(start);
    return st;
}

sknn_status sknn_query(const sknn_index* index, const float* Q, int64_t nq, int32_t k, int32_t* out_idx,
                       float* out_dist, const sknn_options* opt, sknn_stats* stats, sknn_stream_t stream) {
    if (!index) return fail(SKNN_ERR_INVALID_ARG, "index is NULL");
    // Out-of-core queries (the paper partitions Q when it
    // does not fit, "Q in Figure 8 represents one of the partitions"):
    // with host queries and host outputs the queries stream through the device
    // in batches against the resident index; every batch is an independent
    // (exact) query, so the rows are identical to one call.
    const int d = index->t.d;
    if (nq > 0 && Q && out_dist && index->device >= 0 && classify(Q, index->device) == PTR_HOST &&
        classify(out_dist, index->device) == PTR_HOST && (!out_idx || classify(out_idx, index->device) == PTR_HOST)) {
        const sknn_options o = merge_options(opt ? opt : &index->opt);
        int64_t B = o.query_batch;
        if (B <= 0) {
            const size_t free_b = usable_free_bytes(index->device);
            if (free_b == 0) return fail(SKNN_ERR_CUDA, "cudaMemGetInfo failed");
            // per query: input row + output row + clustered copy, center distances and scan state (generous)
            const double per_q = 4.0 * d + 8.0 * k + 2.0 * (4.0 * ((d + 3) & ~3) + 16.0) + 8.0 * k;
            B = (int64_t)((stats ? 0.4 : 0.2) * (double)free_b / per_q);  // two batches in flight without stats
        }
        if (B >= (int64_t)k && B < nq) {
            // SKNN_OOC_SERIAL=1 (study): the serial batch loop also without stats
            // Overlap only when the caller's host buffers are page-locked: measured
            // (tools/ooc_bench.py) with pageable buffers the page-locked staging
            // copies cost more than the overlap gains (C5 443 serial vs 519 ms staged,
            // C2 19 vs 60 ms), so pageable buffers keep the serial loop (the driver
            // stages those copies itself); SKNN_OOC_STAGE=1 forces the staging
            const bool all_pinned = pinned_host(Q) && pinned_host(out_dist) && (!out_idx || pinned_host(out_idx));
            if (!stats && !getenv("SKNN_OOC_SERIAL") && (all_pinned || getenv("SKNN_OOC_STAGE")))
                return query_batches_overlapped(index, Q, nq, k, out_idx, out_dist, opt, B, (cudaStream_t)stream);
            sknn_stats acc;
            memset(&acc, 0, sizeof(acc));
            for (int64_t b0 = 0; b0 < nq; b0 += B) {
                const int64_t nb = std::min(B, nq - b0);
                sknn_stats sb;
                memset(&sb, 0, sizeof(sb));
                sb.struct_size = sizeof(sb);
                SKNN_TRY(run_join(Q + b0 * d, nb, nullptr, index->t.n, d, k, out_idx ? out_idx + b0 * k : nullptr,
                                  out_dist + b0 * k, opt, stats ? &sb : nullptr, (cudaStream_t)stream, index));
                if (!stats) continue;
                // batch sums (sizes and times add up over the batches)
                acc.pairs_total += sb.pairs_total; acc.dist_evals_sparse += sb.dist_evals_sparse;
                acc.dist_evals_dense += sb.dist_evals_dense; acc.dist_evals_brute += sb.dist_evals_brute;
                acc.center_evals += sb.center_evals; acc.cand_pairs += sb.cand_pairs;
                acc.dense_pairs += sb.dense_pairs; acc.dist_recompute += sb.dist_recompute;
                acc.topk_inserts += sb.topk_inserts; acc.rows_loaded += sb.rows_loaded;
                acc.dense_terms = std::max(acc.dense_terms, sb.dense_terms);
                acc.ms_total += sb.ms_total; acc.ms_build_t += sb.ms_build_t; acc.ms_build_q += sb.ms_build_q;
                acc.ms_level1 += sb.ms_level1; acc.ms_sparse += sb.ms_sparse; acc.ms_dense += sb.ms_dense;
                acc.ms_final += sb.ms_final; acc.kernel_launches += sb.kernel_launches;
                acc.mapping_used = sb.mapping_used; acc.path_used = sb.path_used;
                acc.mq += sb.mq; acc.mt = sb.mt;
            }
            if (!stats) return SKNN_OK;
            acc.struct_size = sizeof(acc);
            const size_t sz = stats->struct_size ? std::min(stats->struct_size, sizeof(sknn_stats)) : sizeof(sknn_stats);
            memcpy(stats, &acc, sz);
            return SKNN_OK;
        }
    }
    return run_join(Q, nq, nullptr, index->t.n, d, k, out_idx, out_dist, opt, stats, (cudaStream_t)stream, index);
}

sknn_status sknn_join_indexed(const sknn_index* qindex, const sknn_index* tindex, int32_t k, int32_t* out_idx,
                              float* out_dist, const sknn_options* opt, sknn_stats* stats, sknn_stream_t stream) {
    if (!qindex || !tindex) return fail(SKNN_ERR_INVALID_ARG, "index is NULL");
    if (qindex->t.d != tindex->t.d) return fail(SKNN_ERR_INVALID_ARG, "query and target dimensions differ");
    if (qindex->device != tindex->device) return fail(SKNN_ERR_WRONG_DEVICE, "indexes on different devices");
    return run_join(nullptr, qindex->t.n, nullptr, tindex->t.n, tindex->t.d, k, out_idx, out_dist, opt, stats,
                    (cudaStream_t)stream, tindex, false, qindex);
}

sknn_status sknn_level1_bounds(const sknn_index* qindex, const sknn_index* tindex, int32_t k, const sknn_options* opt,
                               float* ub_out, sknn_stream_t stream) {
    if (!qindex || !tindex || !ub_out) return fail(SKNN_ERR_INVALID_ARG, "NULL pointer");
    if (qindex->t.d != tindex->t.d) return fail(SKNN_ERR_INVALID_ARG, "query and target dimensions differ");
    if (k <= 0 || (int64_t)k > tindex->t.n || k > SKNN_MAX_K) return fail(SKNN_ERR_INVALID_ARG, "bad k");
    DevInfo di;
    SKNN_TRY(device_info(di));
    if (qindex->device != di.device || tindex->device != di.device)
        return fail(SKNN_ERR_WRONG_DEVICE, "index built on another device");
    if (classify(ub_out, di.device) != PTR_DEVICE) return fail(SKNN_ERR_NOT_DEVICE_PTR, "ub_out must be device memory");
    const sknn_options o = merge_options(opt);
    Ctx cx;
    cx.stream = (cudaStream_t)stream;
    cx.device = di.device;
    cx.num_sms = di.num_sms;
    Level1 l1;
    Level1Params lp;
    lp.k = k;
    lp.eta = rounding_eta(tindex->t.d);
    lp.dense_mode = 1;
    lp.ub_in = o.ub_in;
    sknn_status st = run_level1(cx, qindex->t, tindex->t, lp, l1, nullptr);
    if (st == SKNN_OK) {
        cudaError_t e = cudaMemcpyAsync(ub_out, l1.ub, sizeof(float) * qindex->t.m, cudaMemcpyDeviceToDevice, cx.stream);
        if (e != cudaSuccess) st = fail(SKNN_ERR_CUDA, std::string("level-1 bounds copy: ") + cudaGetErrorString(e));
    }
    cx.free_all();
    return st;
}

sknn_status sknn_merge_partials(const int32_t* part_idx, const float* part_d2, int32_t P, int64_t nq, int32_t k,
                                int32_t* out_idx, float* out_dist, int32_t out_squared, sknn_stream_t stream) {
    if (!part_idx || !part_d2 || !out_dist) return fail(SKNN_ERR_INVALID_ARG, "NULL pointer");
    if (P <= 0 || nq < 0 || k <= 0) return fail(SKNN_ERR_INVALID_ARG, "P, k must be > 0 and nq >= 0");
    if (k > SKNN_MAX_K) return fail(SKNN_ERR_UNSUPPORTED, "k > SKNN_MAX_K");
    if (nq == 0) return SKNN_OK;
    DevInfo di;
    SKNN_TRY(device_info(di));
    if (classify(part_idx, di.device) != PTR_DEVICE || classify(part_d2, di.device) != PTR_DEVICE ||
        classify(out_dist, di.device) != PTR_DEVICE || (out_idx && classify(out_idx, di.device) != PTR_DEVICE))
        return fail(SKNN_ERR_NOT_DEVICE_PTR, "sknn_merge_partials takes device pointers only");
    Ctx cx;
    cx.stream = (cudaStream_t)stream;
    cx.device = di.device;
    cx.num_sms = di.num_sms;
    return run_merge(cx, part_idx, part_d2, P, nq, k, out_idx, out_dist, out_squared);
}

sknn_status sknn_merge_partials_ptrs(const int32_t* const* part_idx, const float* const* part_d2, int32_t P,
                                     int64_t nq_total, int64_t row_lo, int64_t nrows, int32_t k, int32_t* out_idx,
                                     float* out_dist, int32_t out_squared, sknn_stream_t stream) {
    if (!part_idx || !part_d2 || !out_dist) return fail(SKNN_ERR_INVALID_ARG, "NULL pointer");
    if (P <= 0 || P > kMaxPeerLists) return fail(SKNN_ERR_INVALID_ARG, "P must be in [1, 16]");
    if (k <= 0 || nq_total < 0 || row_lo < 0 || nrows < 0 || row_lo + nrows > nq_total)
        return fail(SKNN_ERR_INVALID_ARG, "bad k or row range");
    if (k > 32) return fail(SKNN_ERR_UNSUPPORTED, "the peer-list merge keeps k <= 32");
    for (int p = 0; p < P; ++p)
        if (!part_idx[p] || !part_d2[p]) return fail(SKNN_ERR_INVALID_ARG, "NULL list pointer");
    if (nrows == 0) return SKNN_OK;
    DevInfo di;
    SKNN_TRY(device_info(di));
    if (classify(out_dist, di.device) != PTR_DEVICE || (out_idx && classify(out_idx, di.device) != PTR_DEVICE))
        return fail(SKNN_ERR_NOT_DEVICE_PTR, "outputs must be device memory of the current device");
    Ctx cx;
    cx.stream = (cudaStream_t)stream;
    cx.device = di.device;
    cx.num_sms = di.num_sms;
    return run_merge_ptrs(cx, part_idx, part_d2, P, row_lo, nrows, k, out_idx, out_dist, out_squared);
}

sknn_status sknn_index_free(sknn_index* ix) {
    if (!ix) return SKNN_OK;
    int cur = 0;
    cudaGetDevice(&cur);
    if (ix->device != cur) cudaSetDevice(ix->device);
    void* ptrs[] = {ix->t.rows, ix->t.dist, ix->t.orig, ix->t.off, ix->t.centers, ix->t.radius, ix->t.tinfo};
    for (void* p : ptrs)
        if (p) cudaFree(p);
    if (ix->device != cur) cudaSetDevice(cur);
    delete ix;
    return SKNN_OK;
}

sknn_status sknn_index_info(const sknn_index* ix, int64_t* nt, int32_t* d, int32_t* dp, int32_t* mt, int32_t* device) {
    if (!ix) return fail(SKNN_ERR_INVALID_ARG, "index is NULL");
    if (nt) *nt = ix->t.n;
    if (d) *d = ix->t.d;
    if (dp) *dp = ix->t.dp;
    if (mt) *mt = ix->t.m;
    if (device) *device = ix->device;
    return SKNN_OK;
}

sknn_status sknn_index_export(const sknn_index* ix, int32_t* off, int32_t* orig, float* dist, float* centers,
                              float* radius) {
    if (!ix) return fail(SKNN_ERR_INVALID_ARG, "index is NULL");
    const Side& t = ix->t;
    if (off) SKNN_CUDA(cudaMemcpy(off, t.off, sizeof(int32_t) * (t.m + 1), cudaMemcpyDeviceToHost));
    if (orig) SKNN_CUDA(cudaMemcpy(orig, t.orig, sizeof(int32_t) * t.n, cudaMemcpyDeviceToHost));
    if (dist) SKNN_CUDA(cudaMemcpy(dist, t.dist, sizeof(float) * t.n, cudaMemcpyDeviceToHost));
    if (centers) SKNN_CUDA(cudaMemcpy(centers, t.centers, sizeof(float) * t.m * t.dp, cudaMemcpyDeviceToHost));
    if (radius) SKNN_CUDA(cudaMemcpy(radius, t.radius, sizeof(float) * t.m, cudaMemcpyDeviceToHost));
    return SKNN_OK;
}

sknn_status sknn_index_arrays(const sknn_index* ix, void** ptr, size_t* bytes) {
    if (!ix || !ptr || !bytes) return fail(SKNN_ERR_INVALID_ARG, "NULL pointer");
    const Side& t = ix->t;
    void* p[SKNN_INDEX_ARRAYS] = {t.rows, t.dist, t.orig, t.off, t.centers, t.radius, t.tinfo};
    size_t b[SKNN_INDEX_ARRAYS] = {sizeof(float) * (size_t)t.n * t.dp, sizeof(float) * (size_t)t.n,
                                   sizeof(int32_t) * (size_t)t.n, sizeof(int32_t) * (size_t)(t.m + 1),
                                   sizeof(float) * (size_t)t.m * t.dp, sizeof(float) * (size_t)t.m,
                                   sizeof(int4) * (size_t)t.m};
    for (int i = 0; i < SKNN_INDEX_ARRAYS; ++i) {
        ptr[i] = p[i];
        bytes[i] = b[i];
    }
    return SKNN_OK;
}

sknn_status sknn_index_create(int64_t nt, int32_t d, int32_t mt, const sknn_options* opt, sknn_index** out) {
    if (!out) return fail(SKNN_ERR_INVALID_ARG, "out is NULL");
    *out = nullptr;
    if (nt <= 0 || nt >= (int64_t(1) << 31) || d <= 0 || mt <= 0 || mt > nt || mt > kMaxClusters)
        return fail(SKNN_ERR_INVALID_ARG, "bad index geometry");
    DevInfo di;
    SKNN_TRY(device_info(di));
    sknn_index* ix = new (std::nothrow) sknn_index();
    if (!ix) return fail(SKNN_ERR_OOM, "host allocation of the index failed");
    ix->device = di.device;
    ix->user_ptr = nullptr;
    ix->opt = merge_options(opt);
    Side& t = ix->t;
    t.n = nt; t.d = d; t.dp = (d + 3) & ~3; t.m = mt; t.owned = true;
    Ctx cx;
    cx.stream = nullptr;
    cx.device = di.device;
    cx.num_sms = di.num_sms;
    sknn_status st = SKNN_OK;
    do {
        if ((st = cx.alloc_persistent((void**)&t.rows, sizeof(float) * nt * t.dp)) != SKNN_OK) break;
        if ((st = cx.alloc_persistent((void**)&t.dist, sizeof(float) * nt)) != SKNN_OK) break;
        if ((st = cx.alloc_persistent((void**)&t.orig, sizeof(int32_t) * nt)) != SKNN_OK) break;
        if ((st = cx.alloc_persistent((void**)&t.off, sizeof(int32_t) * (mt + 1))) != SKNN_OK) break;
        if ((st = cx.alloc_persistent((void**)&t.centers, sizeof(float) * mt * t.dp)) != SKNN_OK) break;
        if ((st = cx.alloc_persistent((void**)&t.radius, sizeof(float) * mt)) != SKNN_OK) break;
        if ((st = cx.alloc_persistent((void**)&t.tinfo, sizeof(int4) * mt)) != SKNN_OK) break;
        cudaError_t e = cudaStreamSynchronize(nullptr);
        if (e != cudaSuccess) st = fail(SKNN_ERR_CUDA, std::string("index allocation: ") + cudaGetErrorString(e));
    } while (0);
    if (st != SKNN_OK) {
        cx.free_all();
        delete ix;
        return st;
    }
    *out = ix;
    return SKNN_OK;
}

sknn_status sknn_debug_level1(const sknn_index* ix, const float* Q, int64_t nq, int32_t k, const sknn_options* opt,
                              int32_t* mq_out, int32_t* q_cluster, float* ub, int32_t* cand_count, int32_t* cand,
                              int64_t cand_capacity) {
    if (!ix || !Q) return fail(SKNN_ERR_INVALID_ARG, "NULL pointer");
    if (nq <= 0 || k <= 0 || k > ix->t.n || k > SKNN_MAX_K) return fail(SKNN_ERR_INVALID_ARG, "bad nq or k");
    DevInfo di;
    SKNN_TRY(device_info(di));
    sknn_options o = merge_options(opt ? opt : &ix->opt);
    Ctx cx;
    cx.stream = nullptr;
    cx.device = di.device;
    cx.num_sms = di.num_sms;
    sknn_status st = SKNN_OK;
    const Side& ts = ix->t;
    const bool self = index_self_query(o, Q, nq, ix);
    Side qs_local;
    const Side* qs = &ts;
    Level1 l1;
    do {
        const void* dQ;
        bool qh;
        if ((st = stage_in(cx, Q, sizeof(float) * nq * ts.d, &dQ, &qh)) != SKNN_OK) break;
        if (!self) {
            int m = det_lm_num(nq, o.n_clusters_q);
            if ((st = build_side(cx, (const float*)dQ, nq, ts.d, m, o.landmark_trials, o.lloyd_iters, o.seed ^ 0x51ull,
                                 qs_local)) != SKNN_OK)
                break;
            qs = &qs_local;
        }
        Level1Params lp;
        lp.k = k;
        lp.eta = rounding_eta(ts.d);
        lp.dense_mode = 1;  // report the full candidate list in `cand`
        if ((st = run_level1(cx, *qs, ts, lp, l1, nullptr)) != SKNN_OK) break;
        cudaError_t e = cudaStreamSynchronize(nullptr);
        if (e != cudaSuccess) {
            st = fail(SKNN_ERR_CUDA, std::string("level-1 failed: ") + cudaGetErrorString(e));
            break;
        }
        const int mq = qs->m;
        if (mq_out) *mq_out = mq;
        if (ub) cudaMemcpy(ub, l1.ub, sizeof(float) * mq, cudaMemcpyDeviceToHost);
        if (cand_count) cudaMemcpy(cand_count, l1.cand_count, sizeof(int32_t) * mq, cudaMemcpyDeviceToHost);
        if (cand) {
            if (cand_capacity < (int64_t)mq * ts.m) {
                st = fail(SKNN_ERR_INVALID_ARG, "cand_capacity < mq * mt");
                break;
            }
            cudaMemcpy(cand, l1.cand, sizeof(int32_t) * (size_t)mq * ts.m, cudaMemcpyDeviceToHost);
        }
        if (q_cluster) {
            std::string err;
            int32_t* hoff = new int32_t[mq + 1];
            int32_t* horig = new int32_t[nq];
            cudaMemcpy(hoff, qs->off, sizeof(int32_t) * (mq + 1), cudaMemcpyDeviceToHost);
            cudaMemcpy(horig, qs->orig, sizeof(int32_t) * nq, cudaMemcpyDeviceToHost);
            for (int c = 0; c < mq; ++c)
                for (int p = hoff[c]; p < hoff[c + 1]; ++p) q_cluster[horig[p]] = c;
            delete[] hoff;
            delete[] horig;
        }
    } while (0);
    cx.free_all();
    cudaStreamSynchronize(nullptr);
    return st;
}

sknn_status sknn_config_decide(int64_t nq, int64_t nt, int32_t d, int32_t k, const sknn_device_props* props,
                               float r_factor, sknn_config* out) {
    if (!out || nq < 0 || nt <= 0 || d <= 0 || k <= 0) return fail(SKNN_ERR_INVALID_ARG, "bad arguments");
    sknn_device_props p;
    if (props) {
        p = *props;
    } else {
        int dev = 0;
        cudaDeviceProp cp;
        if (cudaGetDevice(&dev) != cudaSuccess || cudaGetDeviceProperties(&cp, dev) != cudaSuccess) {
            cudaGetLastError();
            return fail(SKNN_ERR_CUDA, "no CUDA device to query; pass props");
        }
        p.num_sms = cp.multiProcessorCount;
        p.max_threads_per_sm = cp.maxThreadsPerMultiProcessor;
        p.smem_per_sm = (int)cp.sharedMemPerMultiprocessor;
        p.max_regs_per_thread = 255;
    }
    if (r_factor <= 0.f) r_factor = 0.25f;
    memset(out, 0, sizeof(*out));
    out->th1_bytes = p.smem_per_sm / p.max_threads_per_sm;
    out->th2_bytes = p.max_regs_per_thread * 4;
    int bytes = k * 4;                                        // Fig. 8: k*4 <= th1 -> shared, > th2 -> global
    out->placement = bytes <= out->th1_bytes ? 0 : (bytes > out->th2_bytes ? 2 : 1);
    out->partial_filter = (k > 8 * d) ? 1 : 0;               // P:L615, reading R13
    double maxcur = (double)p.num_sms * p.max_threads_per_sm;
    double rmax = (double)r_factor * maxcur;
    out->r_max_cur = (int64_t)rmax;
    out->tpq_raw = ((double)nq >= rmax || nq == 0) ? 1.0 : rmax / (double)nq;
    int tpq = 1;
    if (out->tpq_raw > 1.0) tpq = 1 << (int)lround(log2(out->tpq_raw));       // reading R15
    out->threads_per_query = tpq;
    const int dp = (d + 3) & ~3;
    out->mapping = (dp <= 32 || k > 32) ? SKNN_MAP_THREAD : SKNN_MAP_WARP;  // B200 rule, see choose_mapping
    out->mq = det_lm_num(std::max<int64_t>(nq, 1), 0);
    out->mt = det_lm_num(nt, 0);
    return SKNN_OK;
}

const char* sknn_error_string(sknn_status s) {
    switch (s) {
        case SKNN_OK: return "SKNN_OK";
        case SKNN_ERR_INVALID_ARG: return "SKNN_ERR_INVALID_ARG";
        case SKNN_ERR_NOT_DEVICE_PTR: return "SKNN_ERR_NOT_DEVICE_PTR";
        case SKNN_ERR_OOM: return "SKNN_ERR_OOM";
        case SKNN_ERR_CUDA: return "SKNN_ERR_CUDA";
        case SKNN_ERR_UNSUPPORTED: return "SKNN_ERR_UNSUPPORTED";
        case SKNN_ERR_WRONG_DEVICE: return "SKNN_ERR_WRONG_DEVICE";
    }
    return "SKNN_ERR_UNKNOWN";
}

const char* sknn_last_error(void) { return g_last_error.c_str(); }

int32_t sknn_version(void) { return (SKNN_VERSION_MAJOR << 16) | SKNN_VERSION_MINOR; }

}  // extern "C"
