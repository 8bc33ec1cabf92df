// sknn_launch.h -- host-side launch context: stream, scratch allocations,
// launch counting and error plumbing of one ABI call. Not part of the ABI.
#pragma once

#include <cuda_runtime.h>
#include <stdint.h>

#include <algorithm>
#include <string>
#include <vector>

#include <nvtx3/nvToolsExt.h>

#include "../../include/sknn.h"
#include "sknn_internal.cuh"

namespace sknn {

void set_last_error(const std::string& msg);

#define SKNN_TRY(expr)                      \
    do {                                    \
        sknn_status _st = (expr);           \
        if (_st != SKNN_OK) return _st;     \
    } while (0)

#define SKNN_CUDA(call)                                                                    \
    do {                                                                                   \
        cudaError_t _e = (call);                                                           \
        if (_e != cudaSuccess) {                                                           \
            ::sknn::set_last_error(std::string(#call) + ": " + cudaGetErrorString(_e));   \
            return _e == cudaErrorMemoryAllocation ? SKNN_ERR_OOM : SKNN_ERR_CUDA;         \
        }                                                                                  \
    } while (0)

// The library's private stream-ordered memory pool of a device (api.cu):
// scratch and index arrays come from it, so its retention policy (up to
// kPoolRetainBytes kept between calls) never touches the device's default
// pool that other users of the process allocate from.
cudaMemPool_t scratch_pool(int device);
// free device memory usable by this library: cudaMemGetInfo's free bytes plus
// the private pool's reserved-but-unused bytes
size_t usable_free_bytes(int device);

// NVTX range around a host-side stage of a call (header-only NVTX v3: no
// link dependency, a no-op unless a tool such as Nsight Systems is attached)
struct NvtxRange {
    explicit NvtxRange(const char* name) { nvtxRangePushA(name); }
    ~NvtxRange() { nvtxRangePop(); }
    NvtxRange(const NvtxRange&) = delete;
    NvtxRange& operator=(const NvtxRange&) = delete;
};

struct Ctx {
    cudaStream_t stream = nullptr;
    int device = 0;
    int num_sms = 148;
    int launches = 0;
    std::vector<void*> scratch;     // freed (stream-ordered) when the call ends
    std::vector<void*> persistent;  // handed to an index, or freed with scratch

    void launched() { ++launches; }

    bool capturing = false;  // recording a CUDA graph: allocations become graph memory nodes
    cudaError_t raw_alloc(void** p, size_t bytes) {
        if (capturing) return cudaMallocAsync(p, bytes, stream);
        return cudaMallocFromPoolAsync(p, bytes, scratch_pool(device), stream);
    }
    sknn_status alloc_scratch(void** p, size_t bytes) {
        if (bytes == 0) bytes = 16;
        cudaError_t e = raw_alloc(p, bytes);
        if (e != cudaSuccess) {
            set_last_error(std::string("cudaMallocAsync(") + std::to_string(bytes) + "): " + cudaGetErrorString(e));
            return SKNN_ERR_OOM;
        }
        scratch.push_back(*p);
        return SKNN_OK;
    }
    sknn_status alloc_persistent(void** p, size_t bytes) {
        if (bytes == 0) bytes = 16;
        cudaError_t e = raw_alloc(p, bytes);
        if (e != cudaSuccess) {
            set_last_error(std::string("cudaMallocAsync(") + std::to_string(bytes) + "): " + cudaGetErrorString(e));
            return SKNN_ERR_OOM;
        }
        persistent.push_back(*p);
        return SKNN_OK;
    }
    sknn_status check_launch(const char* what) {
        cudaError_t e = cudaGetLastError();
        if (e != cudaSuccess) {
            set_last_error(std::string(what) + ": kernel launch failed: " + cudaGetErrorString(e));
            return SKNN_ERR_CUDA;
        }
        return SKNN_OK;
    }
    void free_scratch() {
        for (void* p : scratch) cudaFreeAsync(p, stream);
        scratch.clear();
    }
    void free_all() {
        free_scratch();
        for (void* p : persistent) cudaFreeAsync(p, stream);
        persistent.clear();
    }
};

// k_build.cu
__global__ void k_offsets(const int32_t* __restrict__ counts, int m, int32_t* __restrict__ off,
                          int32_t* __restrict__ cursor);
// Sharded query-side build (target-sharded mode, NEXT-1). mode 1: seeding +
// Lloyd as usual (identical on every rank), then the final assignment of rows
// [lo, hi) only, written to cid_out / dist_out (+ lo) with the centers to
// centers_out; no CSR. mode 2: no clustering -- the centers and the complete
// assignment (cid_in / dist_in, gathered from the ranks) become the side.
struct BuildShard {
    int mode = 0;
    int64_t lo = 0, hi = 0;
    float* centers_out = nullptr;
    int32_t* cid_out = nullptr;
    float* dist_out = nullptr;
    const float* centers_in = nullptr;
    const int32_t* cid_in = nullptr;
    const float* dist_in = nullptr;
};
sknn_status build_side(Ctx& cx, const float* X, int64_t n, int d, int m, int trials, int lloyd, uint64_t seed,
                       Side& out, const BuildShard* shard = nullptr);

// k_assign_tc.cu: nearest-center screen on the tensor cores
bool assign_tc_supported(int dp);
sknn_status run_assign_tc(Ctx& cx, const float* Xp, int64_t n, int dp, const float* centers, int m, int32_t* cid,
                          float* dist, long long* sums, const double* fx, int32_t* counts, int stride = 1);

// k_level1.cu
struct Level1 {
    float* ub = nullptr;          // [mq] inflated calUB per query cluster
    int32_t* cand = nullptr;      // [mq x mt] candidate target clusters, ascending center distance
    int32_t* cand_count = nullptr;  // [mq]
    float* cand_D = nullptr;      // [mq x mt] center distance D(qc, tc) of each sparse candidate
    unsigned long long* work = nullptr;  // [mq] scan work estimate per query (load balancing)
    int4* tiles = nullptr;        // level-2 tasks {query cluster, first member, split | nsplit << 8, part}
    int* ntiles = nullptr;        // [2]: task count, scheduler counter
    int tile = 0;
    int4* merges = nullptr;       // split tiles {query cluster, first member, nsplit, first part}
    int* nmerges = nullptr;       // [1]
    key_t* part = nullptr;        // [split tasks x k x 32] partial lists of split tasks
    unsigned* theta2 = nullptr;   // [nq] shared k-th distance^2 bound of split queries (float bits)
    int32_t* dcand = nullptr;     // [mq x mt] dense-tile candidates (elastic switch), ascending D
    int32_t* dcount = nullptr;    // [mq]
    int2* dtiles = nullptr;       // dense work tiles (128 queries of one cluster)
    int* dntiles = nullptr;       // [2]
    int32_t* owner = nullptr;     // [mq] owning rank of each query cluster (balanced query sharding), or NULL
};
struct DenseOrigin {          // common re-centring point of the dense tiles
    float* o = nullptr;         // [kp] rounded mean target center
    float* cq_o = nullptr;      // [mq] ||c_q - o||
    float* ct_o = nullptr;      // [mt] ||c_t - o||
    float eps = 0.f;            // screen error-bound factor
};
struct Level1Params {
    const DenseOrigin* dorg = nullptr;  // dense screen magnitudes (elastic switch), NULL when unarmed
    int k = 0;
    float eta = 0.f;
    int shard_rank = 0, shard_count = 1;
    int dense_mode = 0;           // 0 auto (cost model), 1 never, 2 every candidate pair
    float dense_tau = 0.5f;       // auto: dense iff |tc| >= 32 and the expected window share >= tau
    const float* ub_in = nullptr; // optional [mq] external upper bounds (min'd with the local calUB)
};
sknn_status run_level1(Ctx& cx, const Side& qs, const Side& ts, const Level1Params& p, Level1& out,
                       Counters* counters);
// balanced query sharding: owner[c] for every query cluster from the level-1
// work estimate (snake deal, heaviest first); zeroes dcount of other ranks' clusters
sknn_status run_shard_owner(Ctx& cx, const Side& qs, Level1& l1, int shard_rank, int shard_count);
// k_dense.cu
struct DenseParams {
    const float* origin = nullptr;
    int k = 0;
    float eta = 0.f;
    key_t* topk_out = nullptr;
    Counters* counters = nullptr;
};
int dense_kp(int dp);
bool dense_supported(int dp);
float dense_eps(int dp);
sknn_status dense_prepare(Ctx& cx, const Side& qs, const Side& ts, DenseOrigin& out);
sknn_status run_dense_tiles(Ctx& cx, const Side& qs, Level1& l1);
sknn_status run_dense(Ctx& cx, const Side& qs, const Side& ts, const Level1& l1, const DenseParams& p);
// k_scan.cu: tiles of `tile` queries of one query cluster (thread-data remapping)
// level-2 task list; slots = resident warps of the scan kernel (scan_resident_warps)
sknn_status run_tiles(Ctx& cx, const Side& qs, int tile, int k, int slots, int shard_rank, int shard_count,
                      Level1& l1, int fig8_width = 1);
int scan_resident_warps(Ctx& cx, int mapping, int dp, int k);
int scan_tile_size(int mapping, int dp, int k);
bool scan_uses_tpq(int mapping, int dp, int k);
bool scan_uses_bigk(int k);

// k_scan.cu
struct ScanParams {
    int k = 0;
    float eta = 0.f;
    int mapping = SKNN_MAP_THREAD;
    int out_squared = 0;
    int64_t index_base = 0;
    int32_t* out_idx = nullptr;
    float* out_dist = nullptr;
    Counters* counters = nullptr;
    const key_t* init_topk = nullptr;    // dense-tile pass results to continue from
};
sknn_status run_scan(Ctx& cx, const Side& qs, const Side& ts, const Level1& l1, const ScanParams& p);
// basic KNN-TI ablation arm (SKNN_MAP_BASIC): thread per query in input order
sknn_status run_scan_basic(Ctx& cx, const Side& qs, const Side& ts, const Level1& l1, const ScanParams& p);
struct ScanArgs;
ScanArgs make_scan_args(const Side& qs, const Side& ts, const Level1& l1, const ScanParams& p);
// k_partial.cu: the paper's partial level-2 filter (SKNN_PATH_PARTIAL); *fell_back
// = true when it did not run (k > 512 or the survivor buffer does not fit)
sknn_status run_partial(Ctx& cx, const Side& qs, const Side& ts, const Level1& l1, const ScanParams& p,
                        bool* fell_back);
sknn_status run_brute(Ctx& cx, const float* Q, int64_t nq, const float* T, int64_t nt, int d, const ScanParams& p);
// dense-only join (k_brute_tiled.cu): register-tiled SIMT contraction + fused top-k
sknn_status run_brute_tiled(Ctx& cx, const float* Q, int64_t nq, int ldq, const float* T, int64_t nt, int ldt,
                            const int32_t* torig, int d, const ScanParams& p);
// dimensions from which auto takes the dense-only path (measured)
constexpr int kDenseOnlyDp = 1024;
sknn_status run_merge(Ctx& cx, const int32_t* part_idx, const float* part_d2, int P, int64_t nq, int k,
                      int32_t* out_idx, float* out_dist, int out_squared);
// merge of P lists in separate (possibly peer) buffers, rows [row_lo, row_lo + nrows)
constexpr int kMaxPeerLists = 16;
sknn_status run_merge_ptrs(Ctx& cx, const int32_t* const* part_idx, const float* const* part_d2, int P,
                           int64_t row_lo, int64_t nrows, int k, int32_t* out_idx, float* out_dist, int out_squared);

}  // namespace sknn
