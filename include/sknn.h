/*
 * sknn.h -- C ABI of the B200-native Sweet KNN exact KNN join.
 *
 * Method: Chen, Ding, Shen, "Sweet KNN: An Efficient KNN on GPU through
 * Reconciliation between Redundancy Removal and Regularity", ICDE 2017.
 * Citations "P:L<n>" refer to line n of the paper transcript with
 * the section / equation / algorithm / figure the line falls in.
 *
 * The operation (every entry point below computes or serves it):
 *   KNN join ("KNN join problem"; Fig. 4 main procedure P:L271):
 *   for every query point q in Q, the k points of the target set T closest
 *   to q in Euclidean distance. Results are exact: the triangle-
 *   inequality (TI) filters only skip targets that provably cannot be among
 *   the k nearest. Ties are broken by the lowest
 *   target index; every output row is sorted ascending by (distance, index)
 *   (readings R2, R4). Squared distances are accumulated in fp32 in
 *   the fixed dimension order c = 0..d-1; distances are IEEE sqrt of those.
 *
 * Memory conventions (all entry points):
 *   - Point sets are row-major, contiguous, fp32: Q is [nq x d], T is [nt x d].
 *   - Outputs: out_idx [nq x k] int32 original target row indices (plus
 *     opt->index_base), out_dist [nq x k] fp32 Euclidean distances (or
 *     squared distances when opt->out_squared != 0).
 *   - Pointers may be DEVICE pointers (on the current CUDA device) or HOST
 *     pointers (pageable or pinned). Host inputs are staged to the device and
 *     host outputs copied back inside the call; in that case the call
 *     synchronises `stream` before returning. With device pointers only, the
 *     call is stream-ordered: it enqueues all work on `stream` and returns
 *     without waiting (unless stats are requested); results are valid once
 *     `stream` completes.
 *   - The library never frees caller memory. Scratch is allocated from a
 *     private stream-ordered memory pool of the device (cudaMallocFromPoolAsync
 *     on `stream`; up to 8 GB of freed scratch stays reserved in that pool
 *     between calls, the device's default pool is not touched) and released
 *     (stream-ordered) before return.
 *   - sknn_join / sknn_join_ex with device pointers and no stats: when the
 *     same (device, pointers, sizes, options) repeat, the second call records
 *     the join into a CUDA graph and later calls replay it (one launch); the
 *     replay reads the CURRENT contents of the recorded buffers, so results
 *     are always those of the data at call time (opt->use_graph = -1 opts out).
 *   - `stream` is a cudaStream_t (NULL = the legacy default stream).
 *
 * Errors: every function returns an sknn_status; no C++ exception crosses the
 * ABI. On error the outputs are unspecified and sknn_last_error() (thread-
 * local) holds a one-line description. Inputs must be finite (NaN/Inf are
 * undefined behaviour).
 */
#ifndef SKNN_H_
#define SKNN_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define SKNN_VERSION_MAJOR 0
#define SKNN_VERSION_MINOR 1

/* cudaStream_t without pulling in the CUDA headers. */
typedef struct CUstream_st* sknn_stream_t;

typedef enum {
    SKNN_OK = 0,
    SKNN_ERR_INVALID_ARG = -1,    /* null pointer, nq < 0, nt <= 0, d <= 0, k <= 0, k > nt, nt >= 2^31, bad option */
    SKNN_ERR_NOT_DEVICE_PTR = -2, /* pointer on another device / unrecognised memory */
    SKNN_ERR_OOM = -3,            /* device or host allocation failed */
    SKNN_ERR_CUDA = -4,           /* a CUDA runtime call or kernel launch failed */
    SKNN_ERR_UNSUPPORTED = -5,    /* device is not sm_100, or k > SKNN_MAX_K */
    SKNN_ERR_WRONG_DEVICE = -6    /* index used on a device other than the one that built it */
} sknn_status;

/* Largest k supported (the paper's largest, Fig. 10 / Table V).
 * kNearests placement follows Fig. 8: shared memory for
 * k*4 <= th1, registers for k <= 32, shared memory with fewer threads per CTA
 * beyond. k > 32 uses the thread-per-query scan only (no dense tiles, no
 * brute-force path). */
#define SKNN_MAX_K 512

/* Execution-path override (sknn_options.force_path). */
enum {
    SKNN_PATH_AUTO = 0,   /* adaptive scheme (Fig. 8 re-derived for B200)                 */
    SKNN_PATH_SPARSE = 1, /* TI filters + point-level scan only (Alg. 1 + Alg. 2)          */
    SKNN_PATH_DENSE = 2,  /* TI filters; every surviving cluster pair on the dense tile path */
    SKNN_PATH_BRUTE = 3,  /* no filtering: every query against every target (the anchor and */
                          /* the dense-only path): register-tiled SIMT contraction with a    */
                          /* fused top-k, k <= 32; auto takes it at dp >= 1024 for sknn_join */
                          /* and sknn_query (the index's permuted rows), where the TI filters */
                          /* keep most pairs (Table IV arcene / dorothea)         */
    SKNN_PATH_PARTIAL = 4 /* TI filters; PARTIAL level-2 filter (§IV-B1): theta   */
                          /* fixed at the level-1 UB, every window member's distance stored  */
                          /* in a global survivor buffer, then a k-selection kernel; k <= 512 */
                          /* (falls back to the full filter when the buffer would not fit in */
                          /* half of the free device memory). It reads the survivor count    */
                          /* back to size that buffer: the call synchronises `stream` (the   */
                          /* one host round trip of the library; never taken by auto)         */
};

/* Level-2 thread mapping override (sknn_options.mapping), §IV-B2 / §IV-D3. */
enum {
    SKNN_MAP_AUTO = 0,
    SKNN_MAP_THREAD = 1,  /* one thread per query ("query level parallelism")       */
    SKNN_MAP_WARP = 2,    /* one warp per query ("multi-level parallelism")         */
    SKNN_MAP_BASIC = 3    /* ablation arm: the basic KNN-TI Sweet KNN starts from     */
                          /* (Fig. 4 / Alg. 2): one thread per */
                          /* query in INPUT order (no thread-data remapping, §IV-C1), */
                          /* every member of a candidate cluster visited from the top */
                          /* (Alg. 2's continue / break), kNearests a sorted array in */
                          /* thread-local memory; sparse only, k <= 32, no sharding.  */
                          /* Same exact result as every other mapping    */
};

/* Tunables. Zero-initialise and set struct_size = sizeof(sknn_options), or
 * call sknn_options_default(). A NULL options pointer means all defaults. */
typedef struct {
    size_t struct_size;       /* ABI versioning: sizeof(sknn_options) of the caller              */
    int32_t n_clusters_q;     /* 0 = auto floor(3*sqrt(nq)), clamped to [1, min(nq, 8192)] */
    int32_t n_clusters_t;     /* 0 = auto floor(3*sqrt(nt)), same clamp                           */
    int32_t landmark_trials;  /* 0 = 10 trials of the landmark sampler                   */
    int32_t lloyd_iters;      /* -1 = default 2 (north_star "a few Lloyd iterations", reading R9); 0 = paper sampler only */
    uint64_t seed;            /* landmark sampler seed (results never depend on it)               */
    int32_t force_path;       /* SKNN_PATH_*                                                       */
    int32_t mapping;          /* SKNN_MAP_*                                                        */
    float dense_threshold;    /* elastic switch threshold (0 = auto)                               */
    float r_factor;           /* cache-conflict factor r (0 = 0.25)                        */
    int32_t out_squared;      /* 1: out_dist holds squared distances (for partial-list exchange)  */
    int32_t pad0;
    int64_t index_base;       /* added to every output index (target-sharded global indices)      */
    int32_t shard_rank;       /* query sharding: only query clusters c with c % shard_count ==    */
    int32_t shard_count;      /*   shard_rank are processed (0/1 = all); other output rows untouched */
    int64_t query_batch;      /* sknn_query with HOST queries and outputs (out-of-core, the paper's */
                              /*   query partitions P:L575): queries per device batch; 0 = auto   */
                              /*   (all at once when they fit in 40% of the free device memory)   */
    int32_t self_query;       /* sknn_query / sknn_debug_level1: is Q the index's build set (reuse */
                              /*   its clustering for the query side, a self-join)?        */
                              /*   1 = yes (caller asserts Q holds the build rows), -1 = never,     */
                              /*   0 = auto: yes iff Q is the SAME POINTER and size as the build    */
                              /*   input -- the build buffer must then still be alive and unchanged */
                              /*   (a freed-and-reused address would silently answer for old rows) */
    int32_t pad1;
    const float* ub_in;       /* optional DEVICE [mq] upper bounds of the query clusters' k-th    */
                              /*   distance (e.g. sknn_level1_bounds of every target shard, min  */
                              /*   over ranks); level-1 takes min(its calUB, ub_in[qc]). Only    */
                              /*   meaningful with the query side of sknn_join_indexed / the same */
                              /*   query clustering; rows may then hold fewer than k real entries */
                              /*   (placeholders: distance +inf, index -1) -- for partial lists  */
    int32_t use_graph;        /* sknn_join_ex on device pointers without stats: 0 = auto (replay a */
                              /*   captured CUDA graph of the whole join when the same shapes,     */
                              /*   pointers and options repeat), -1 = never                         */
    int32_t shard_policy;     /* query sharding (shard_count > 1): which query clusters a rank owns. */
                              /*   0 = interleave (c % shard_count == shard_rank);                   */
                              /*   1 = balanced: every rank runs level-1 over ALL query clusters      */
                              /*   (replicated) and deals the clusters, heaviest first by |qc| x the */
                              /*   level-1 scan-work estimate, to ranks in snake order -- identical  */
                              /*   on every rank (deterministic clustering and integer work sums)     */
} sknn_options;

/* Counters and per-stage times of one call (filled only when a non-NULL
 * pointer is passed; the call then synchronises `stream` before returning). */
typedef struct {
    size_t struct_size;
    uint64_t pairs_total;          /* nq * nt                                                         */
    uint64_t dist_evals_sparse;    /* point distances evaluated by the level-2 scan ("count") */
    uint64_t dist_evals_dense;     /* query-target pairs covered by dense tiles                       */
    uint64_t dist_evals_brute;     /* pairs evaluated by the brute-force path                         */
    uint64_t center_evals;         /* query-to-candidate-center distances in level-2 (Alg. 2 line 6)  */
    uint64_t cand_pairs;           /* surviving (query cluster, target cluster) pairs after level-1  */
    uint64_t dense_pairs;          /* of which processed as dense tiles                               */
    uint64_t dist_recompute;       /* dense-tile survivors recomputed with the exact fp32 formula     */
    float ms_total;                /* CUDA-event time of the whole call on `stream`                   */
    float ms_build_t, ms_build_q, ms_level1, ms_sparse, ms_dense, ms_final;
    int32_t mapping_used;          /* SKNN_MAP_THREAD or SKNN_MAP_WARP                               */
    int32_t path_used;             /* SKNN_PATH_*                                                     */
    int32_t mq, mt;                /* cluster counts used                                             */
    int32_t kernel_launches;       /* kernels this call launched                                      */
    int32_t pad0;
    uint64_t topk_inserts;         /* kNearests updates by the level-2 scan (P:L453 update overhead)   */
    uint64_t rows_loaded;          /* target rows fetched by the level-2 scan: once per warp for the  */
                                   /*   warp-union walk, once per evaluation otherwise (§8(d) bytes)  */
    uint32_t dense_terms;          /* bf16 MMA terms per K-step of the dense tiles: 1 = exact integer */
                                   /*   tiles (hi parts only), 2-3 = split-precision screen; 0 = none */
    uint32_t pad1;
} sknn_stats;

/* Opaque resident target index (sknn_build / sknn_query). Owns device memory:
 * the target points permuted into cluster order, padded to a multiple of 4
 * floats, their distances to the cluster centers (descending within each
 * cluster), original indices, cluster offsets, centers and radii. */
typedef struct sknn_index sknn_index;

/* Adaptive-scheme decisions (Fig. 8, §IV-D) for a problem on a device. */
typedef struct {
    int32_t num_sms, max_threads_per_sm, smem_per_sm, max_regs_per_thread;
} sknn_device_props;

typedef struct {
    int32_t th1_bytes;        /* smem/SM / max threads/SM                   */
    int32_t th2_bytes;        /* max regs/thread * 4                        */
    int32_t placement;        /* 0 shared, 1 registers, 2 global (Fig. 8)            */
    int32_t partial_filter;   /* 1 iff k/d > 8 (reading R13)                 */
    int64_t r_max_cur;        /* r * max_cur total threads                  */
    double tpq_raw;           /* r*max_cur/|Q| or 1                     */
    int32_t threads_per_query;/* nearest power of two in log2 (reading R15), uncapped */
    int32_t mapping;          /* SKNN_MAP_THREAD / SKNN_MAP_WARP chosen for B200      */
    int32_t mq, mt;           /* cluster counts floor(3*sqrt(n)) clamped              */
} sknn_config;

/* ---------------------------------------------------------------- API --- */

/* Fill *opt with defaults (struct_size set). */
void sknn_options_default(sknn_options* opt);

/* KNN join of Q against T (Fig. 4 main procedure): clusters both
 * sets (Step 1; Q == T with nq == nt is a self-join and is
 * clustered once, as in the paper's experiments P:L697), filters cluster
 * pairs (Step 2, Alg. 1), filters and evaluates points
 * (Step 3, Alg. 2), and writes the k nearest of every query.
 * out_idx may be NULL ("w/ or w/o index information"). nq == 0 is a
 * no-op returning SKNN_OK. */
sknn_status sknn_join(const float* Q, int64_t nq, const float* T, int64_t nt,
                      int32_t d, int32_t k, int32_t* out_idx, float* out_dist,
                      sknn_stream_t stream);

/* sknn_join with options (NULL = defaults) and optional stats (NULL = none). */
sknn_status sknn_join_ex(const float* Q, int64_t nq, const float* T, int64_t nt,
                         int32_t d, int32_t k, int32_t* out_idx, float* out_dist,
                         const sknn_options* opt, sknn_stats* stats,
                         sknn_stream_t stream);

/* Build a resident target index (Step 1 for T). T may be device
 * or host memory; the index keeps its own copy. The index records the value
 * of the T pointer: a later sknn_query with Q == that pointer and nq == nt is
 * treated as a self-join (the caller must not have changed the contents). */
sknn_status sknn_build(const float* T, int64_t nt, int32_t d,
                       const sknn_options* opt, sknn_index** out,
                       sknn_stream_t stream);

/* Query a resident index: Step 1 for Q, then Steps 2-3 (Fig. 4 lines 3-6).
 * The index is read-only: concurrent queries on different streams are safe.
 * Must run on the device that built the index (else SKNN_ERR_WRONG_DEVICE).
 * Out-of-core (the paper's query partitions): when Q, out_dist and
 * out_idx (if given) are all HOST memory, the queries stream through the
 * device in batches of opt->query_batch rows (0 = auto from the free device
 * memory), each batch an independent exact query, so results equal one call;
 * stats are summed over the batches. The call synchronises `stream`. */
sknn_status sknn_query(const sknn_index* index, const float* Q, int64_t nq,
                       int32_t k, int32_t* out_idx, float* out_dist,
                       const sknn_options* opt, sknn_stats* stats,
                       sknn_stream_t stream);

/* Sharded clustering of one point set (target-sharded mode: every rank holds
 * all of Q; NEXT-1 "sharded Q clustering"). sknn_cluster_count: the m that
 * sknn_build / the functions below use for n points (floor(3 sqrt(n)),
 * clamped; opt->n_clusters_t overrides). sknn_build_assign_shard runs the
 * landmark sampler and the Lloyd passes over all of T (deterministic: every
 * rank computes the same centers) and the FINAL assignment of rows
 * [row_lo, row_hi) only (row_lo % 8 == 0), writing centers_out [m x dp]
 * (dp = d rounded up to 4), cid_out[row] and dist_out[row] (exact fp32
 * member distances) for those rows; device pointers. After the ranks'
 * rows are gathered, sknn_build_from_assignment turns the complete
 * assignment into an index -- CSR, member sort, cluster summaries -- equal
 * to the one sknn_build returns for the same T and options (P:L241,
 * P:L317-331). Both synchronise `stream`. */
int32_t sknn_cluster_count(int64_t n, const sknn_options* opt);
sknn_status sknn_build_assign_shard(const float* T, int64_t nt, int32_t d, const sknn_options* opt,
                                    int64_t row_lo, int64_t row_hi, float* centers_out,
                                    int32_t* cid_out, float* dist_out, sknn_stream_t stream);
sknn_status sknn_build_from_assignment(const float* T, int64_t nt, int32_t d, const sknn_options* opt,
                                       const float* centers, int32_t m, const int32_t* cid,
                                       const float* dist, sknn_index** out, sknn_stream_t stream);

/* Merge P partial result lists into one (multi-GPU target-sharded mode;
 * the paper's merge of per-thread sorted heaps, generalised to
 * ranks). part_idx [P x nq x k] int32 global indices, part_d2 [P x nq x k]
 * fp32 SQUARED distances, each row sorted ascending by (d2, idx) (as written
 * by sknn_query with out_squared = 1). Output: the k smallest (d2, idx) keys
 * of each query over all P lists; out_dist gets sqrt(d2) unless
 * out_squared != 0. Any P >= 1 and k <= SKNN_MAX_K (one warp per query,
 * bitonic merge of sorted lists). Device pointers only. */
sknn_status sknn_merge_partials(const int32_t* part_idx, const float* part_d2,
                                int32_t P, int64_t nq, int32_t k,
                                int32_t* out_idx, float* out_dist,
                                int32_t out_squared, sknn_stream_t stream);

/* The same merge reading the P lists from P separate buffers -- the fused
 * peer-memory merge of the target-sharded mode (NEXT-1): rank r passes the
 * device addresses of every rank's [nq_total x k] partial lists as mapped
 * into its own address space (symmetric memory / CUDA IPC over NVLink; local
 * buffers work the same) and merges its rows [row_lo, row_lo + nrows) into
 * out_idx / out_dist [nrows x k], the remote lists read directly by the merge
 * kernel -- no exchange collective. part_idx / part_d2 are HOST arrays of P
 * pointers (1 <= P <= 16); the pointers are not classified (peer addresses
 * belong to other devices); k <= 32. The caller orders the peers' writes
 * before this call (e.g. a symmetric-memory barrier on `stream`). */
sknn_status sknn_merge_partials_ptrs(const int32_t* const* part_idx, const float* const* part_d2,
                                     int32_t P, int64_t nq_total, int64_t row_lo, int64_t nrows,
                                     int32_t k, int32_t* out_idx, float* out_dist,
                                     int32_t out_squared, sknn_stream_t stream);

/* Free an index (after all queries using it completed). NULL is a no-op. */
sknn_status sknn_index_free(sknn_index* index);

/* Index geometry: points, dimension, padded dimension, clusters, device. */
sknn_status sknn_index_info(const sknn_index* index, int64_t* nt, int32_t* d,
                            int32_t* dp, int32_t* mt, int32_t* device);

/* Copy index metadata to HOST buffers (any may be NULL; synchronous):
 * off [mt+1] cluster offsets into the permuted order, orig [nt] original row
 * of each permuted point, dist [nt] distance to its center (descending within
 * a cluster, ties by index ascending, P:L241 / reading R11), centers
 * [mt x dp], radius [mt] (max member distance, 0 for an empty cluster). */
sknn_status sknn_index_export(const sknn_index* index, int32_t* off, int32_t* orig,
                              float* dist, float* centers, float* radius);

/* Device arrays of an index (no copy): the build-once-and-share path of the
 * multi-GPU query-sharded mode ("rank 0 builds and broadcasts
 * it", e.g. ncclBroadcast over NVLink). ptr[i] / bytes[i] for i in
 * SKNN_INDEX_ARRAY_*; the arrays stay owned by the index. Writing into them is
 * allowed only for an index made by sknn_index_create and before any query. */
enum {
    SKNN_INDEX_ARRAY_ROWS = 0,    /* [nt x dp] fp32 points in cluster order        */
    SKNN_INDEX_ARRAY_DIST = 1,    /* [nt] fp32 member-to-center distance          */
    SKNN_INDEX_ARRAY_ORIG = 2,    /* [nt] int32 original row index                 */
    SKNN_INDEX_ARRAY_OFF = 3,     /* [mt+1] int32 cluster offsets                  */
    SKNN_INDEX_ARRAY_CENTERS = 4, /* [mt x dp] fp32                                */
    SKNN_INDEX_ARRAY_RADIUS = 5,  /* [mt] fp32                                     */
    SKNN_INDEX_ARRAY_TINFO = 6,   /* [mt] int4 {lo, hi, radius bits, min dist bits} */
    SKNN_INDEX_ARRAYS = 7
};
sknn_status sknn_index_arrays(const sknn_index* index, void** ptr, size_t* bytes);

/* An index of the given geometry with allocated but UNINITIALISED arrays on
 * the current device, to be filled through sknn_index_arrays with the arrays
 * of an index built elsewhere (same nt, d, mt; e.g. broadcast from rank 0).
 * opt is stored as the index's default options (NULL = defaults). The index
 * has no build input pointer: self-joins through it need
 * sknn_options.self_query = 1. */
sknn_status sknn_index_create(int64_t nt, int32_t d, int32_t mt, const sknn_options* opt,
                              sknn_index** out);

/* Join of two prebuilt indexes: the query index (sknn_build over Q, whose
 * clustering is then reused, P:L241 Step 1 for Q) against the target index
 * (Steps 2-3, Fig. 4 lines 3-6). Output rows in the query index's original row
 * order. This is the target-sharded mode's building block: every rank clusters
 * Q identically (seeded), exchanges level-1 bounds (sknn_level1_bounds) and
 * joins with opt->ub_in = the minimum over ranks. Device outputs. */
sknn_status sknn_join_indexed(const sknn_index* qindex, const sknn_index* tindex, int32_t k,
                              int32_t* out_idx, float* out_dist, const sknn_options* opt,
                              sknn_stats* stats, sknn_stream_t stream);

/* Level-1 upper bounds (calUB) of every query cluster of qindex
 * against tindex: ub_out DEVICE [mq] (mq = sknn_index_info(qindex).mt),
 * +inf for an empty query cluster. Each value bounds the k-th nearest
 * distance of every member of the cluster among tindex's points, hence among
 * any superset of them (the minimum over target shards is a global bound). */
sknn_status sknn_level1_bounds(const sknn_index* qindex, const sknn_index* tindex, int32_t k,
                               const sknn_options* opt, float* ub_out, sknn_stream_t stream);

/* Level-1 products of a query against an index, to HOST buffers (testing):
 * q_cluster [nq] cluster of each query, ub [mq] the inflated upper bound of
 * each query cluster (calUB), cand_count [mq] surviving target
 * clusters (groupFilter, Alg. 1), cand [mq x mt] candidate target clusters
 * in ascending center distance (first cand_count[i] of row i valid). Any
 * output may be NULL. mq_out receives the query cluster count. */
sknn_status sknn_debug_level1(const sknn_index* index, const float* Q, int64_t nq,
                              int32_t k, const sknn_options* opt, int32_t* mq_out,
                              int32_t* q_cluster, float* ub, int32_t* cand_count,
                              int32_t* cand, int64_t cand_capacity);

/* Adaptive-scheme decisions (Fig. 8, §IV-D) -- pure host arithmetic.
 * props == NULL queries the current device. */
sknn_status sknn_config_decide(int64_t nq, int64_t nt, int32_t d, int32_t k,
                               const sknn_device_props* props, float r_factor,
                               sknn_config* out);

const char* sknn_error_string(sknn_status status);
const char* sknn_last_error(void);   /* thread-local message of the last failure */
int32_t sknn_version(void);          /* (major << 16) | minor */

#ifdef __cplusplus
}
#endif
#endif /* SKNN_H_ */
