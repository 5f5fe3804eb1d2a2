/*
 * omp_baseline.c -- CPU SPEED baseline for bench.py (SURVEY §8(d) "CPU speed
 * baseline"): the same two computations as the oracle, parallelised with
 * OpenMP over all host cores.  NOT the oracle (oracle/ is the plain single-thread
 * checker) and NOT part of the GPU product path; it shares no code with either.
 *
 *  omp_csr_to_csc : counting sort of the CSR into CSC (untimed preparation)
 *  omp_spmspv     : y = A x over plus-times, fp64, the "SpMSpV-bucket" column
 *                   merge (Azad & Bulu\c{c}, IPDPS'17): threads scan slices of x and
 *                   append (row, a_ij x_j) to row-range buckets, then each bucket
 *                   is merged in a thread-private dense accumulator and its
 *                   touched rows sorted; output ascending by row (Alg 2,
 *                   PAPER.md P:358-366, parallel form)
 *  omp_bfs        : level-synchronous top-down BFS (Alg 3 levels):
 *                   per-thread next-frontier buffers, vertices claimed with a
 *                   compare-and-swap on their level
 * Build: gcc -O3 -fopenmp -shared -fPIC omp_baseline.c -o libomp_baseline.so
 */
#include <omp.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

int omp_max_threads(void) { return omp_get_max_threads(); }

int omp_csr_to_csc(int64_t m, int64_t n, const int64_t *row_ptr, const int32_t *col_idx, const double *val,
                   int64_t *col_ptr, int32_t *row_idx, double *cval) {
    const int64_t nnz = row_ptr[m];
    memset(col_ptr, 0, (size_t)(n + 1) * sizeof(int64_t));
    for (int64_t p = 0; p < nnz; ++p) col_ptr[col_idx[p] + 1]++;
    for (int64_t j = 0; j < n; ++j) col_ptr[j + 1] += col_ptr[j];
    int64_t *pos = (int64_t *)malloc((size_t)(n + 1) * sizeof(int64_t));
    if (!pos) return 2;
    memcpy(pos, col_ptr, (size_t)(n + 1) * sizeof(int64_t));
    for (int64_t i = 0; i < m; ++i)
        for (int64_t p = row_ptr[i]; p < row_ptr[i + 1]; ++p) {
            const int64_t q = pos[col_idx[p]]++;
            row_idx[q] = (int32_t)i;
            if (val && cval) cval[q] = val[p];
        }
    free(pos);
    return 0;
}

typedef struct {
    int32_t row;
    double v;
} pair_t;

static int cmp_i32(const void *a, const void *b) {
    const int32_t x = *(const int32_t *)a, y = *(const int32_t *)b;
    return (x > y) - (x < y);
}

/* y_idx / y_val must hold m entries.  Returns 0, or 2 on allocation failure. */
int omp_spmspv(int64_t m, int64_t n, const int64_t *col_ptr, const int32_t *row_idx, const double *val, int64_t k,
               const int32_t *x_idx, const double *x_val, int32_t *y_idx, double *y_val, int64_t *y_nnz,
               int nthreads) {
    (void)n;
    if (nthreads <= 0) nthreads = omp_get_max_threads();
    const int nb = nthreads * 4;
    const int64_t span = (m + nb - 1) / nb;
    int64_t *cnt = (int64_t *)calloc((size_t)nthreads * nb + 1, sizeof(int64_t));
    int64_t *ycnt = (int64_t *)calloc((size_t)nb + 1, sizeof(int64_t));
    if (!cnt || !ycnt) return 2;
    /* pass 1: entries per (thread, bucket) */
#pragma omp parallel num_threads(nthreads)
    {
        const int t = omp_get_thread_num();
        int64_t *c = cnt + (size_t)t * nb;
#pragma omp for schedule(static)
        for (int64_t e = 0; e < k; ++e) {
            const int32_t j = x_idx[e];
            for (int64_t p = col_ptr[j]; p < col_ptr[j + 1]; ++p) c[row_idx[p] / span]++;
        }
    }
    /* offsets, bucket-major then thread */
    int64_t *off = (int64_t *)malloc(((size_t)nthreads * nb + 1) * sizeof(int64_t));
    int64_t *bstart = (int64_t *)malloc(((size_t)nb + 1) * sizeof(int64_t));
    if (!off || !bstart) return 2;
    int64_t tot = 0;
    for (int b = 0; b < nb; ++b) {
        bstart[b] = tot;
        for (int t = 0; t < nthreads; ++t) {
            off[(size_t)t * nb + b] = tot;
            tot += cnt[(size_t)t * nb + b];
        }
    }
    bstart[nb] = tot;
    pair_t *buf = (pair_t *)malloc((size_t)(tot > 0 ? tot : 1) * sizeof(pair_t));
    if (!buf) return 2;
    /* pass 2: scatter (row, a x) into the buckets (same static schedule) */
#pragma omp parallel num_threads(nthreads)
    {
        const int t = omp_get_thread_num();
        int64_t *o = off + (size_t)t * nb;
#pragma omp for schedule(static)
        for (int64_t e = 0; e < k; ++e) {
            const int32_t j = x_idx[e];
            const double xj = x_val ? x_val[e] : 1.0;
            for (int64_t p = col_ptr[j]; p < col_ptr[j + 1]; ++p) {
                const int32_t r = row_idx[p];
                pair_t *q = &buf[o[r / span]++];
                q->row = r;
                q->v = (val ? val[p] : 1.0) * xj;
            }
        }
    }
    /* pass 3: merge each bucket in a private dense accumulator over its row span */
    int32_t **rows_b = (int32_t **)calloc((size_t)nb, sizeof(int32_t *));
    double **vals_b = (double **)calloc((size_t)nb, sizeof(double *));
    if (!rows_b || !vals_b) return 2;
    int fail = 0;
#pragma omp parallel num_threads(nthreads)
    {
        double *acc = (double *)malloc((size_t)span * sizeof(double));
        unsigned char *seen = (unsigned char *)calloc((size_t)span, 1);
        if (!acc || !seen) fail = 1;
#pragma omp for schedule(dynamic, 1)
        for (int b = 0; b < nb; ++b) {
            if (fail) continue;
            const int64_t r0 = (int64_t)b * span;
            const int64_t len = bstart[b + 1] - bstart[b];
            int32_t *tr = (int32_t *)malloc((size_t)(len > 0 ? len : 1) * sizeof(int32_t));
            int64_t nt = 0;
            for (int64_t q = bstart[b]; q < bstart[b + 1]; ++q) {
                const int64_t r = buf[q].row - r0;
                if (!seen[r]) {
                    seen[r] = 1;
                    acc[r] = 0.0;
                    tr[nt++] = (int32_t)r;
                }
                acc[r] += buf[q].v;
            }
            qsort(tr, (size_t)nt, sizeof(int32_t), cmp_i32);
            double *tv = (double *)malloc((size_t)(nt > 0 ? nt : 1) * sizeof(double));
            for (int64_t i = 0; i < nt; ++i) {
                tv[i] = acc[tr[i]];
                seen[tr[i]] = 0;
                tr[i] += (int32_t)r0;
            }
            rows_b[b] = tr;
            vals_b[b] = tv;
            ycnt[b] = nt;
        }
        free(acc);
        free(seen);
    }
    if (fail) return 2;
    int64_t ytot = 0;
    for (int b = 0; b < nb; ++b) {
        const int64_t c = ycnt[b];
        ycnt[b] = ytot;
        ytot += c;
    }
    ycnt[nb] = ytot;
#pragma omp parallel for num_threads(nthreads) schedule(static)
    for (int b = 0; b < nb; ++b) {
        const int64_t c = ycnt[b + 1] - ycnt[b];
        memcpy(y_idx + ycnt[b], rows_b[b], (size_t)c * sizeof(int32_t));
        memcpy(y_val + ycnt[b], vals_b[b], (size_t)c * sizeof(double));
        free(rows_b[b]);
        free(vals_b[b]);
    }
    *y_nnz = ytot;
    free(rows_b);
    free(vals_b);
    free(buf);
    free(off);
    free(bstart);
    free(cnt);
    free(ycnt);
    return 0;
}

/* levels: int32[n] out (-1 unreachable).  Edge u -> i for every stored A_iu
 * (column u of A = out-neighbours of u under y = A x). */
int omp_bfs(int64_t n, const int64_t *col_ptr, const int32_t *row_idx, int64_t source, int32_t *levels,
            int nthreads) {
    if (nthreads <= 0) nthreads = omp_get_max_threads();
    int32_t *front = (int32_t *)malloc((size_t)(n > 0 ? n : 1) * sizeof(int32_t));
    int32_t *next = (int32_t *)malloc((size_t)(n > 0 ? n : 1) * sizeof(int32_t));
    if (!front || !next) return 2;
#pragma omp parallel for num_threads(nthreads) schedule(static)
    for (int64_t v = 0; v < n; ++v) levels[v] = -1;
    levels[source] = 0;
    front[0] = (int32_t)source;
    int64_t nf = 1;
    int32_t L = 0;
    while (nf > 0) {
        int64_t nn = 0;
#pragma omp parallel num_threads(nthreads)
        {
            int32_t local[1024];
            int nl = 0;
#pragma omp for schedule(dynamic, 64)
            for (int64_t f = 0; f < nf; ++f) {
                const int32_t u = front[f];
                for (int64_t p = col_ptr[u]; p < col_ptr[u + 1]; ++p) {
                    const int32_t i = row_idx[p];
                    int32_t expect = -1;
                    if (__atomic_load_n(&levels[i], __ATOMIC_RELAXED) == -1 &&
                        __atomic_compare_exchange_n(&levels[i], &expect, L + 1, 0, __ATOMIC_RELAXED,
                                                    __ATOMIC_RELAXED)) {
                        local[nl++] = i;
                        if (nl == 1024) {
                            const int64_t o = __atomic_fetch_add(&nn, nl, __ATOMIC_RELAXED);
                            memcpy(next + o, local, (size_t)nl * sizeof(int32_t));
                            nl = 0;
                        }
                    }
                }
            }
            if (nl) {
                const int64_t o = __atomic_fetch_add(&nn, nl, __ATOMIC_RELAXED);
                memcpy(next + o, local, (size_t)nl * sizeof(int32_t));
            }
        }
        int32_t *t = front;
        front = next;
        next = t;
        nf = nn;
        ++L;
    }
    free(front);
    free(next);
    return 0;
}
