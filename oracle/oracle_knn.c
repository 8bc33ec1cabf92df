/*
 * oracle_knn.c -- TEST INFRASTRUCTURE ONLY.
 *
 * Plain, slow, obviously-correct CPU brute-force KNN join: the definition the
 * Sweet KNN method (Chen, Ding, Shen, ICDE 2017) must reproduce exactly.
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
 * --impl reference legs may load this library. It shares no code with the
 * CUDA path under paper_conf_icde_chends17_b200/csrc.
 *
 * What it computes (paper problem statement PAPER.md
 * L17-35 "KNN join", Fig. 4 output R at P:L271; distance = Euclidean):
 *
 *   D2(i,j)     = sum_{c=0}^{d-1} (Q[i,c] - T[j,c])^2      (fp64, c ascending)
 *   NN(i)       = the k indices j with the lexicographically smallest keys
 *                 (D2(i,j), j), in ascending key order      (ties -> lowest j,
 *                 DESIGN.md reading R2; order of R, reading R4)
 *   out_idx[i,r]  = j_r
 *   out_dist[i,r] = (float) sqrt(D2(i, j_r))
 *
 * Method: for every query a bounded max-heap of size k keyed by (D2, j), then
 * a sort of the k survivors. OpenMP over queries. Compile with
 * -O2 -fopenmp -ffp-contract=off (no fast-math).
 *
 * Parity pins: tests/test_oracle.py (hand cases P1-P4, numpy lexsort brute
 * force, scipy cKDTree, invariants O2).
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#ifdef _OPENMP
#include <omp.h>
#endif

typedef struct {
    double d2;
    int64_t j;
} key_t_;

/* a < b in the (d2, j) lexicographic order */
static int key_less(key_t_ a, key_t_ b) {
    if (a.d2 < b.d2) return 1;
    if (a.d2 > b.d2) return 0;
    return a.j < b.j;
}

/* max-heap on key_less */
static void sift_down(key_t_* h, int n, int i) {
    for (;;) {
        int l = 2 * i + 1, r = l + 1, m = i;
        if (l < n && key_less(h[m], h[l])) m = l;
        if (r < n && key_less(h[m], h[r])) m = r;
        if (m == i) return;
        key_t_ t = h[i]; h[i] = h[m]; h[m] = t;
        i = m;
    }
}

static void sift_up(key_t_* h, int i) {
    while (i > 0) {
        int p = (i - 1) / 2;
        if (!key_less(h[p], h[i])) return;
        key_t_ t = h[i]; h[i] = h[p]; h[p] = t;
        i = p;
    }
}

static int cmp_key(const void* a, const void* b) {
    key_t_ x = *(const key_t_*)a, y = *(const key_t_*)b;
    if (key_less(x, y)) return -1;
    if (key_less(y, x)) return 1;
    return 0;
}

/* Squared Euclidean distance, fp64, dimensions in ascending order. */
static double sq_dist(const float* a, const float* b, int d) {
    double s = 0.0;
    for (int c = 0; c < d; ++c) {
        double diff = (double)a[c] - (double)b[c];
        s += diff * diff;
    }
    return s;
}

/*
 * Returns 0 on success, -1 on invalid arguments (k > nt, k <= 0, d <= 0).
 * Q: [nq x d] row-major fp32, T: [nt x d] row-major fp32 (host memory).
 * out_idx: [nq x k] int32 (may be NULL), out_dist: [nq x k] fp32,
 * out_d2: optional [nq x k] fp64 exact-ish squared distances (may be NULL).
 * nthreads <= 0 means the OpenMP default.
 */
int oracle_knn_join(const float* Q, int64_t nq, const float* T, int64_t nt,
                    int d, int k, int32_t* out_idx, float* out_dist,
                    double* out_d2, int nthreads) {
    if (nq < 0 || nt <= 0 || d <= 0 || k <= 0 || (int64_t)k > nt) return -1;
#ifdef _OPENMP
    if (nthreads > 0) omp_set_num_threads(nthreads);
#else
    (void)nthreads;
#endif
    int err = 0;
#pragma omp parallel
    {
        key_t_* heap = (key_t_*)malloc(sizeof(key_t_) * (size_t)k);
        if (!heap) {
#pragma omp atomic write
            err = 1;
        }
#pragma omp for schedule(dynamic, 16)
        for (int64_t i = 0; i < nq; ++i) {
            if (!heap) continue;
            const float* q = Q + i * (int64_t)d;
            int n = 0;
            for (int64_t j = 0; j < nt; ++j) {
                key_t_ kk;
                kk.d2 = sq_dist(q, T + j * (int64_t)d, d);
                kk.j = j;
                if (n < k) {
                    heap[n] = kk;
                    sift_up(heap, n);
                    ++n;
                } else if (key_less(kk, heap[0])) {
                    heap[0] = kk;
                    sift_down(heap, n, 0);
                }
            }
            qsort(heap, (size_t)n, sizeof(key_t_), cmp_key);
            for (int r = 0; r < k; ++r) {
                if (out_idx) out_idx[i * k + r] = (int32_t)heap[r].j;
                out_dist[i * k + r] = (float)sqrt(heap[r].d2);
                if (out_d2) out_d2[i * k + r] = heap[r].d2;
            }
        }
        free(heap);
    }
    return err ? -2 : 0;
}

/* Number of threads OpenMP would use (for reporting "cores"). */
int oracle_num_threads(void) {
#ifdef _OPENMP
    return omp_get_max_threads();
#else
    return 1;
#endif
}
