/*
 * tsmv.h -- C ABI of libtsmv.so: tiled sparse matrix - sparse vector
 * multiplication (TileSpMSpV) and direction-optimising TileBFS on NVIDIA B200
 * (sm_100a).
 *
 * Method: Ji, Song, Lu, Jin, Tan, Liu, "TileSpMSpV: A Tiled Algorithm for
 * Sparse Matrix-Sparse Vector Multiplication on GPUs", ICPP '22.
 * "P:n" = line n of the paper text; "R<k>" = reading k in DESIGN.md.
 *
 * Conventions for every entry point
 *  - No C++ exception crosses the ABI; every call returns a tsmv_status.  On a
 *    non-OK status a thread-local message is available from tsmv_last_error().
 *  - Pointers marked "host or device" are classified per call with
 *    cudaPointerGetAttributes: device (or managed) memory is used in place,
 *    host memory (pageable or pinned) is staged through ctx-owned device
 *    buffers with the copies enqueued on the caller's stream.
 *  - A context is bound to one CUDA device and is not thread-safe.  All work
 *    is enqueued on the `cuda_stream` argument (a cudaStream_t; NULL = the
 *    legacy default stream).
 *  - Index types: row pointers int64, column / row / vertex ids int32 (so
 *    n < 2^31), counts int64.
 */
#ifndef TSMV_H
#define TSMV_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct tsmv_ctx tsmv_ctx; /* opaque */

typedef enum {
    TSMV_OK = 0,
    TSMV_EINVAL = 1,      /* bad argument (sizes, NULL, unsorted/duplicate x, source range) */
    TSMV_ENOMEM = 2,      /* device or host allocation failed */
    TSMV_ECUDA = 3,       /* a CUDA runtime error (message in tsmv_last_error) */
    TSMV_ENCCL = 4,       /* NCCL unavailable or a collective failed (message in tsmv_last_error) */
    TSMV_ECAPACITY = 5,   /* y_cap < y_nnz: *y_nnz holds the required size */
    TSMV_EUNSUPPORTED = 6 /* valid request this build does not support */
} tsmv_status;

typedef enum { TSMV_F64 = 0, TSMV_F32 = 1, TSMV_PATTERN = 2 } tsmv_dtype;

/* Semirings of y = A x (P:157-160 problem statement; Boolean AND = x, OR = +).
 *  PLUS_TIMES : y_i = sum_j a_ij * x_j.  F32 matrices: fp32 storage, fp64
 *               accumulation, one rounding at the end (R3).  PATTERN: a_ij = 1.
 *  OR_AND     : structural product only; y_val is not written (may be NULL).
 *  MIN_SECOND : y_i = min_j x_j over stored a_ij (a_ij ignored); with x_j = j
 *               this yields the minimum-id parent of BFS. */
typedef enum { TSMV_PLUS_TIMES = 0, TSMV_OR_AND = 1, TSMV_MIN_SECOND = 2 } tsmv_semiring;

/* TileBFS kernels (Sec 3.4): Push-CSC (Alg 5), Push-CSR (Alg 6),
 * Pull-CSC (Alg 7); AUTO applies the per-level rule of reading R9. */
typedef enum {
    TSMV_DIR_AUTO = 0,
    TSMV_DIR_PUSH_CSC = 1,
    TSMV_DIR_PUSH_CSR = 2,
    TSMV_DIR_PULL_CSC = 3
} tsmv_dir;

typedef struct {
    int32_t device;              /* CUDA ordinal the context lives on */
    int32_t tile_dim;            /* nt in {16, 32, 64}; default 16 */
    int32_t sparse_tile_max_nnz; /* tiles with <= this many nonzeros go to the side
                                    matrix (R12); default 2; 0 = none */
    int32_t build_bfs;           /* 1 = also build the TileBFS bitmask tiles (square A);
                                    default 1 when nrows == ncols and nranks == 1;
                                    2 = a 2D-partition block A_ij (any shape, nranks 1):
                                    the structures serve tsmv_bfs2d_expand only */
    double push_csr_density;     /* |F|/n threshold Push-CSC -> Push-CSR; the paper's is 0.01
                                    (P:1423-1433); default 0.05, measured on B200 */
    double pull_alpha;           /* Pull-CSC when m_f > m_u / alpha (R9); Beamer's 14; default 2,
                                    measured on B200 (list-driven Push-CSC levels stay cheaper than
                                    bitmap-wide levels longer than on the paper's GPU) */
    int32_t force_dir;           /* tsmv_dir; AUTO = rule of R9 (tests / ablation) */
    int32_t rank, nranks;        /* row-block partition: this rank / number of ranks (1 = single GPU) */
    int64_t row_begin;           /* global id of local row 0 (multiple of 64 when nranks > 1) */
    const int64_t *row_splits;   /* host, nranks+1 global row boundaries (NULL when nranks == 1);
                                    copied by tsmv_create */
    const void *nccl_unique_id;  /* host, 128 bytes from tsmv_nccl_unique_id on one rank, the same on
                                    every rank, or NULL.  When set, tsmv_create
                                    creates the context's own NCCL communicator (collective over the
                                    nranks ranks, each on its own GPU; nranks == 1 allowed) and
                                    tsmv_bfs / tsmv_spmspv become collective calls that exchange the
                                    frontier / x themselves.  When NULL with nranks > 1, the caller
                                    drives the exchange with the tsmv_bfs_dist_* primitives. */
    double row_driven_density;   /* nt = 16: x density k / ncols at or above which tsmv_spmspv runs the
                                    row-driven kernel (Alg 4: every row tile walks its
                                    tiles, skipping those whose x segment misses them) instead of the
                                    column-driven one, for matrices that keep <= 10 % of their
                                    nonzeros in the side matrix and <= 32 per tile (small matrices:
                                    at any density); 0 = never.  Results are identical; default 0.05,
                                    the crossover measured on B200. */
    double pull_alpha_burst;     /* (r2) alpha used instead of pull_alpha on a level whose frontier
                                    grew >= burst_growth x over the previous level's (the explosive
                                    levels of low-diameter graphs, where Beamer's 14 pays: R-MAT s26
                                    290 -> 387 GTEPS), R9'; default 14; 0 = off */
    double burst_growth;         /* growth factor of that test; default 4 (grids and bands grow
                                    < 4x per level and keep pull_alpha) */
} tsmv_options;

/* Per-call counters of the last tsmv_spmspv (read from device on request). */
typedef struct {
    int64_t x_nnz;          /* k */
    int64_t x_segments;     /* non-empty nt-segments of x */
    int64_t tile_items;     /* tiles in the tile columns of non-empty segments (a3) */
    int64_t side_items;     /* side-matrix nonzeros in the columns of x (a5) */
    int64_t y_nnz;
    int64_t hit_tiles;      /* tiles whose column mask intersects the segment mask */
    int64_t hit_columns;    /* (tile, column) pairs in both the tile's and x's masks */
    int64_t tile_macs;      /* useful multiply-adds inside tiles (side ones = side_items) */
    int64_t tile_macs_indirect; /* of tile_macs, those whose value / index came from the
                                   nonzero arrays (not inline in the 64-byte tile record) */
} tsmv_call_stats;

/* Built-format census. */
typedef struct {
    int64_t nrows, ncols, nnz;
    int32_t tile_dim;
    int32_t symmetric;          /* pattern symmetric (detected; BFS then keeps one bitmask copy) */
    int64_t n_tiles;            /* non-empty tiles (before extraction) */
    int64_t n_dense_tiles;      /* tiles kept in tile format (> sparse_tile_max_nnz nnz) */
    int64_t dense_nnz;          /* nonzeros in tile format */
    int64_t side_nnz;           /* nonzeros in the side matrix */
    int64_t bytes_spmspv;       /* device bytes of the SpMSpV structures */
    int64_t bytes_bfs;          /* device bytes of the BFS bitmask structures */
    int64_t bytes_workspace;    /* accumulators, bitmaps, scratch */
    double build_ms;            /* device time of tsmv_create's builder */
} tsmv_info;

/* Size of the per-level arrays of tsmv_bfs_stats.  It is NOT a traversal limit:
 * a traversal with more levels runs to completion (every level written to
 * `levels`); only the first TSMV_MAX_LEVELS entries of the per-level arrays are
 * filled. */
#define TSMV_MAX_LEVELS 65536
typedef struct {
    int32_t nlevels;                 /* number of non-empty levels (source level counts) */
    int64_t reached;                 /* vertices with level >= 0 (global) */
    int64_t edges_traversed;         /* sum of out-degrees of reached vertices (R16) */
    double ms;                       /* device time source-init -> last level */
    int32_t dir_per_level[TSMV_MAX_LEVELS];       /* tsmv_dir used to expand level L */
    int64_t frontier_per_level[TSMV_MAX_LEVELS];  /* |F| of level L */
    float level_ms[TSMV_MAX_LEVELS];              /* device time of level L: from the decision
                                                     to expand L (%globaltimer) to the decision
                                                     for L + 1 (the last level: to the end);
                                                     the paper's per-level analysis, Fig 10
                                                      */
} tsmv_bfs_stats;

/* Fill *opt with the defaults documented above.  Never fails for non-NULL opt. */
tsmv_status tsmv_default_options(tsmv_options *opt);

/* Bootstrap of a distributed context: a new ncclUniqueId written
 * to out128 (128 bytes, host).  Call on ONE rank and hand the bytes to the others
 * (e.g. torch.distributed.broadcast_object_list), then every rank passes them as
 * tsmv_options.nccl_unique_id to tsmv_create.  NCCL is loaded at run time
 * (libnccl.so.2; TSMV_NCCL_LIB overrides).  Errors: EINVAL (NULL), ENCCL. */
tsmv_status tsmv_nccl_unique_id(void *out128);

/* Build the tiled representation of A (Sec 3.2.1; BFS bitmasks
 * Sec 3.2.3) on opt->device.
 *   nrows, ncols : local rows (rows of this rank's block) and global columns.
 *   row_ptr      : int64[nrows+1], host or device; row_ptr[0] must be 0.
 *   col_idx      : int32[nnz], host or device; ascending and unique within each row,
 *                  in [0, ncols).
 *   values       : nnz values (double for F64, float for F32), host or device;
 *                  must be NULL iff dtype == TSMV_PATTERN.
 *   opt          : NULL = defaults.
 * The ctx deep-copies everything; the caller may free its inputs on return.
 * Errors: EINVAL (sizes, tile_dim, unsorted/duplicate/out-of-range columns),
 * ENOMEM, ECUDA.  *out is NULL on failure. */
tsmv_status tsmv_create(tsmv_ctx **out, int64_t nrows, int64_t ncols, const int64_t *row_ptr,
                        const int32_t *col_idx, const void *values, tsmv_dtype dtype,
                        const tsmv_options *opt);

/* y = A x over `sr` (Sec 3.3, Fig 4).
 *   x_nnz, x_idx, x_val : the sparse x; x_idx int32 UNIQUE global column ids in any
 *                  order (R21: ascending input takes the fast path; otherwise the
 *                  call sorts x once on the device), host or device; x_val double
 *                  (F64/PATTERN) or float (F32), host or device, may be NULL for OR_AND.
 *                  Distributed context with a communicator (nccl_unique_id): a
 *                  COLLECTIVE call; each rank passes the x entries it owns (indices
 *                  in its row range [row_splits[rank], row_splits[rank+1]) of the
 *                  square A, ascending), the call exchanges them (count all-gather +
 *                  grouped broadcasts) and returns y for the rank's own rows.
 *   y_cap, y_idx, y_val : caller-owned outputs (host or device).  y_idx int32
 *                  ascending GLOBAL row ids; y_val same type as x_val (not written
 *                  for OR_AND; may then be NULL).  y_cap >= nrows always suffices.
 *   y_nnz        : host out; set even on ECAPACITY (contents of y then unspecified).
 * The call synchronises `cuda_stream` once (to return y_nnz).
 * Errors: EINVAL (unsorted / duplicate / out-of-range x, semiring/dtype mismatch),
 * ECAPACITY, ECUDA.  On EINVAL the ctx workspaces stay clean. */
tsmv_status tsmv_spmspv(tsmv_ctx *c, tsmv_semiring sr, int64_t x_nnz, const int32_t *x_idx,
                        const void *x_val, int64_t y_cap, int32_t *y_idx, void *y_val,
                        int64_t *y_nnz, void *cuda_stream);

/* Asynchronous variant for pipelines and benchmarks: same semantics, but every
 * pointer must be device memory, nothing is synchronised, and the result size is
 * written to *y_nnz_dev (device int64) when the stream reaches it: y_nnz, or -1
 * if x was invalid (the workspaces stay clean).  If y_nnz > y_cap only the first
 * y_cap entries are written.  x_nnz must be >= 1. */
tsmv_status tsmv_spmspv_async(tsmv_ctx *c, tsmv_semiring sr, int64_t x_nnz, const int32_t *x_idx,
                              const void *x_val, int64_t y_cap, int32_t *y_idx, void *y_val,
                              int64_t *y_nnz_dev, void *cuda_stream);

/* Per-kernel device timing of tsmv_spmspv* (CUDA events recorded on the call's
 * stream around each of its three kernels).  tsmv_set_timing(c, 1) starts a new
 * window; tsmv_get_timing waits for the events and returns the summed ms of
 * {x-scan, expand, compact, whole call} over the `calls` timed calls since. */
tsmv_status tsmv_set_timing(tsmv_ctx *c, int32_t enable);

/* Retune the TileBFS direction rule (reading R9) of a built context:
 * the tsmv_options fields push_csr_density (> 0), pull_alpha (> 0) and force_dir
 * (TSMV_DIR_AUTO .. TSMV_DIR_PULL_CSC) for the next traversals.  EINVAL on range. */
tsmv_status tsmv_set_direction_rule(tsmv_ctx *c, double push_csr_density, double pull_alpha, int32_t force_dir);
tsmv_status tsmv_get_timing(tsmv_ctx *c, double *ms_out4, int64_t *calls);

/* Development trace of the multiply phase: when `device_buffer` (u64 words,
 * tsmv_trace_words(c) of them, device memory, caller-owned) is set, every warp of
 * every later SpMSpV call writes 8 words {phase-B start ns, chunk-loop end ns,
 * chunks, ns in tile chunks, ns in side chunks, longest chunk ns, barrier arrival
 * ns, multiplies}.  NULL disables. */
tsmv_status tsmv_set_trace(tsmv_ctx *c, void *device_buffer);
int64_t tsmv_trace_words(const tsmv_ctx *c);

/* Counters of the last tsmv_spmspv on this ctx (synchronous D2H read). */
tsmv_status tsmv_last_call_stats(tsmv_ctx *c, tsmv_call_stats *s);

/* TileBFS from `source` (Alg 3 P:418-430 with the three kernels of Sec 3.4,
 * P:1417-1628).  Single-GPU contexts, and distributed contexts with their own
 * communicator (nccl_unique_id): then a COLLECTIVE call (same source on every
 * rank; levels = the rank's own rows; stats global and identical on every rank;
 * one in-place broadcast of each rank's owned frontier words per level, the
 * statistics computed from the replicated frontier, no reduction).  Distributed
 * contexts without a communicator use the tsmv_bfs_dist_* calls.  Requires a
 * square A built with build_bfs.
 *   levels : int32[nrows] host or device out: hop count from source, -1 if
 *            unreachable (R15).
 *   stats  : host, may be NULL.
 * Returns after the traversal (stream synchronised).  Errors: EINVAL (source
 * out of range, not square, no BFS structures), ECUDA. */
tsmv_status tsmv_bfs(tsmv_ctx *c, int64_t source, int32_t *levels, tsmv_bfs_stats *stats,
                     void *cuda_stream);

/* BFS tree over the min-second semiring (the semiring the paper
 * lists for BFS-type SpMSpV).  Given the levels of a
 * finished tsmv_bfs on this ctx, writes
 *   parents[v] = min { u : A[v][u] stored (edge u -> v) and levels[u] == levels[v] - 1 },
 *   parents[source] = source, parents[v] = -1 when levels[v] == -1,
 * i.e. what Alg 3 yields with x_j = j over MIN_SECOND: a unique,
 * Graph500-valid tree.
 *   levels  : int32[nrows] device, as written by tsmv_bfs (not modified).
 *   parents : int32[nrows] device out, caller-owned.
 * Enqueued on cuda_stream, not synchronised.  Single-GPU contexts with BFS
 * structures only.  Errors: EINVAL (NULL, host pointers, distributed ctx, no
 * BFS structures), ECUDA. */
tsmv_status tsmv_bfs_parents(tsmv_ctx *c, const int32_t *levels, int32_t *parents, void *cuda_stream);

/* Multi-source TileBFS: Alg 3 from nsrc
 * sources at once, the multiple-BFS workload of P:171-177.  One bit per source in
 * 64-bit vertex words; every level is one bottom-up (Pull-CSC, Alg 7) pass for all
 * sources over the row structure (tile row words gather the frontier words of
 * the tile's column segment) and the side CSR.
 *   nsrc    : 1..64.
 *   sources : host int64[nsrc], each in [0, nrows) (repeats allowed).
 *   levels  : device int32[nrows * nsrc], vertex-major: levels[v * nsrc + s] =
 *             hop count of v from sources[s], -1 if unreachable (R15 per source).
 *   stats   : host, may be NULL: nlevels = max over sources of the non-empty
 *             levels, pairs_reached = sum over sources of reached vertices,
 *             edges_traversed = sum over sources of R16, ms = device time.
 * Single-GPU contexts with BFS structures and tile_dim 16 only (else EINVAL /
 * EUNSUPPORTED).  Returns after the traversal (stream synchronised). */
typedef struct {
    int32_t nlevels;
    int64_t pairs_reached;
    int64_t edges_traversed;
    double ms;
} tsmv_msbfs_stats;
tsmv_status tsmv_msbfs(tsmv_ctx *c, int32_t nsrc, const int64_t *sources, int32_t *levels,
                       tsmv_msbfs_stats *stats, void *cuda_stream);

/* ---- distributed TileBFS, caller-driven exchange (row-block partition, SURVEY
 * §8(e) / DESIGN.md §8; contexts WITHOUT a communicator: simulated ranks, gloo) ----
 * Each rank owns global rows [row_splits[rank], row_splits[rank+1]).  Per level:
 *   tsmv_bfs_dist_expand  -> this rank's newly discovered owned vertices as a bitmap
 *                            segment (uint32 words, bit v%32 of word (v-row_begin)/32);
 *   caller all-gathers the segments (torch.distributed / NCCL), each padded to
 *   `stride_words` words, in rank order;
 *   tsmv_bfs_dist_merge   -> OR the gathered frontier into the replicated visited
 *                            bitmap, clear the old frontier, return the statistics.
 * (r2) begin / merge return this rank's SHARES out_stats[3] = { |F| of its own rows,
 * m_f share (sum of the GLOBAL out-degrees of its frontier vertices), m_u local (sum
 * of the in-degrees of its unvisited rows) }, computed over its own rows only
 * (O(n / P) per level); the caller sums the three over the ranks and passes
 * tsmv_choose_dir(...) of the sums as `dir` (1..3) to expand, so every rank takes
 * the same decision.  The global out-degrees (column counts of all blocks) are set
 * once with tsmv_bfs_dist_set_degrees (a one-rank context uses its own).  levels:
 * device memory, int32[local rows].  All ranks make the same calls in the same order. */
tsmv_status tsmv_bfs_dist_set_degrees(tsmv_ctx *c, const int32_t *outdeg_global /* int32[ncols], host or device */);
tsmv_status tsmv_bfs_dist_begin(tsmv_ctx *c, int64_t source, int32_t *levels, int64_t *out_stats,
                                void *cuda_stream);
/* dir: TSMV_DIR_PUSH_CSC .. TSMV_DIR_PULL_CSC, optionally | TSMV_DIST_WIDE: a hint
 * for a late Pull-CSC level (few unvisited edges left: m_u < nnz / 4), which then
 * tests 32 row tiles' visited words per warp; the result is the same. */
#define TSMV_DIST_WIDE 0x100
tsmv_status tsmv_bfs_dist_expand(tsmv_ctx *c, int32_t dir, uint32_t *owned_words_out, void *cuda_stream);
/* merge: out_stats may be host memory (the call synchronises, as begin does) or
 * device memory (int64[3] written on the stream, no synchronisation: the caller
 * all-reduces m_f / m_u on the device and reads the level's result once). */
tsmv_status tsmv_bfs_dist_merge(tsmv_ctx *c, const uint32_t *gathered, int64_t stride_words,
                                int64_t *out_stats, void *cuda_stream);
/* Words of this rank's owned segment = ceil((row_splits[r+1]-row_splits[r])/32). */
int64_t tsmv_owned_words(const tsmv_ctx *c);

/* ---- 2D-partitioned TileBFS steps (Alg 3 P:418-430 with the
 * OR-AND semiring of P:1373-1379; DESIGN.md §8 "2D") ----
 * Rank (i, j) of a Pr x Pc grid holds A_ij = A[R_i, C_j] as an ordinary context
 * (nranks = 1, local row ids 0..|R_i|-1, local column ids of C_j's padded column
 * space).  A level: y = A_ij x_j by tsmv_spmspv(_async) with TSMV_OR_AND, then
 *   tsmv_bfs2d_scatter : y's local row ids (y_idx[0 .. *y_nnz), device, *y_nnz on
 *       the device, at most y_cap read) -> bitmap words[nwords] over R_i (zeroed
 *       first; bit r % 32 of word r / 32); nwords >= ceil(rows / 32);
 *   caller: all-to-all in processor row i of the words of each sub-piece R_ij';
 *   tsmv_bfs2d_merge : OR of nseg partial bitmaps segs[p * stride_words + w] of this
 *       rank's nverts = |R_ij| vertices; new = OR & ~visited; visited |= new;
 *       levels[v] = level for new v; front_out[w] = new words; stats_dev (device
 *       int64[3], no synchronisation) = { |new|, sum outdeg[v], sum indeg[v] } over
 *       the new v (outdeg / indeg int32[nverts] of this rank's vertices, GLOBAL
 *       degrees, may be NULL: sum 0) -- the shares of Alg 3's |F|, m_f and the m_u
 *       decrement, summed over the ranks by the caller;
 *   caller: all-gather in processor column j of the front words -> C_j's bitmap;
 *   tsmv_bfs2d_list : bitmap words (nbits bits) -> ascending ids idx_out[0..count);
 *       count_out host (the call synchronises the stream) or device.
 * Direction-optimising levels (context built with build_bfs = 2) replace the
 * SpMSpV + scatter by
 *   tsmv_bfs2d_expand : dir 1..3 (| TSMV_DIST_WIDE for late pull levels), decided
 *       by the caller from the summed statistics (tsmv_choose_dir); x_words = C_j's
 *       frontier bitmap (ceil(ncols / 32) words), row_new (may be NULL) = R_i's
 *       bitmap of the vertices found by the previous level (the processor-row
 *       all-gather of the owners' front words) ORed into visited_rows first;
 *       visited_rows = R_i's visited bitmap (ceil(nrows / 32) words; the pull level
 *       tests and the discoveries update it); next_words = the partial bitmap of
 *       R_i found by this block (zeroed first; the all-to-all send buffer);
 *       levels_rows int32[nrows] scratch (discoveries write level + 1).
 *       Push-CSC (Alg 5), Push-CSR (Alg 6) and Pull-CSC (Alg 7) run the level kernels
 *       of the row-block path on the block's own tiles.
 * All buffers are the caller's device memory; the context supplies the device, the
 * stream's scratch (bfs2d_list) and the SM count.  Errors: EINVAL on NULL / host
 * pointers or inconsistent sizes. */
tsmv_status tsmv_bfs2d_scatter(tsmv_ctx *c, const int32_t *y_idx, const int64_t *y_nnz, int64_t y_cap,
                               uint32_t *words, int64_t nwords, void *cuda_stream);
tsmv_status tsmv_bfs2d_merge(tsmv_ctx *c, const uint32_t *segs, int32_t nseg, int64_t stride_words,
                             int64_t nverts, uint32_t *visited, int32_t *levels, int32_t level,
                             uint32_t *front_out, const int32_t *outdeg, const int32_t *indeg,
                             int64_t *stats_dev, void *cuda_stream);
tsmv_status tsmv_bfs2d_expand(tsmv_ctx *c, int32_t dir, const uint32_t *x_words, const uint32_t *row_new,
                              uint32_t *visited_rows, uint32_t *next_words, int32_t *levels_rows,
                              int32_t level, void *cuda_stream);
tsmv_status tsmv_bfs2d_list(tsmv_ctx *c, const uint32_t *words, int64_t nbits, int32_t *idx_out,
                            int64_t *count_out, void *cuda_stream);

/* Direction rule of reading R9: PULL_CSC if m_f > m_u / alpha,
 * else PUSH_CSR if frontier / n >= push_csr_density, else PUSH_CSC; force_dir wins
 * when not AUTO.  alpha = pull_alpha_burst when prev_frontier > 0 and frontier >=
 * burst_growth x prev_frontier (reading R9', r2), else pull_alpha; prev_frontier =
 * |F| of the previous level (0 or negative: unknown).  opt NULL = defaults. */
int32_t tsmv_choose_dir(const tsmv_options *opt, int64_t n, int64_t frontier, int64_t m_f, int64_t m_u,
                        int64_t prev_frontier);

/* Census of the built format (host out). */
tsmv_status tsmv_get_info(const tsmv_ctx *c, tsmv_info *info);

/* Rebuild CSR from the tiled structures (tiles + side matrix), host outputs:
 * row_ptr int64[nrows+1], col_idx int32[nnz], values (type of the ctx; NULL
 * allowed).  Used by the round-trip test of the builder. */
tsmv_status tsmv_export_csr(tsmv_ctx *c, int64_t *row_ptr, int32_t *col_idx, void *values);

/* Export the TileBFS bitmask tiles in the paper's presentation (Fig 5,
 * P:770-788): orient 0 = A1 column words, 1 = A2 row words, MSB-first bits,
 * tiles listed in (J, I) order for A1 and (I, J) for A2, side-matrix entries
 * folded back in.  Host outputs of capacity max_tiles (EINVAL if exceeded). */
tsmv_status tsmv_export_bitmask_tiles(tsmv_ctx *c, int32_t orient, int64_t max_tiles,
                                      int64_t *tile_I, int64_t *tile_J, uint64_t *words,
                                      int64_t *n_tiles);

/* Free everything the ctx owns.  NULL-safe. */
tsmv_status tsmv_destroy(tsmv_ctx *c);

/* Thread-local message for the last non-OK status ("" if none). */
const char *tsmv_last_error(void);

/* ABI version, (major << 16) | minor. */
int32_t tsmv_version(void);

#ifdef __cplusplus
}
#endif
#endif /* TSMV_H */
