// common.cuh -- internal definitions of libtsmv.so (not part of the ABI).
//
// Layout of the tiled matrix in HBM (DESIGN.md §"Data layout"):
//   TileSet = one "tile-CSC": non-empty nt x nt tiles grouped by tile column
//   (P:481-503 stores them "in the CSR format" by tile row; we keep the
//   column-grouped twin because the vector-driven kernels walk tile columns,
//   P:1439-1457), structure-of-arrays so that the intersection step reads only
//   the 2..8-byte column masks of the tiles it tests.
#pragma once
#include <cstdint>
#include <cstdio>
#include <cstring>
#include <string>
#include <vector>
#include <cuda_runtime.h>
#include "../../include/tsmv.h"

#define TSMV_VERSION ((1 << 16) | 0)

namespace tsmv {

// ------------------------------------------------------------------ errors
void set_error(const char *fmt, ...);

struct Err {
    tsmv_status st;
};

#define TSMV_CUDA(call)                                                                 \
    do {                                                                                \
        cudaError_t _e = (call);                                                        \
        if (_e != cudaSuccess) {                                                        \
            ::tsmv::set_error("%s:%d %s: %s", __FILE__, __LINE__, #call,                \
                              cudaGetErrorString(_e));                                  \
            throw ::tsmv::Err{_e == cudaErrorMemoryAllocation ? TSMV_ENOMEM : TSMV_ECUDA}; \
        }                                                                               \
    } while (0)

#define TSMV_REQUIRE(cond, ...)                 \
    do {                                        \
        if (!(cond)) {                          \
            ::tsmv::set_error(__VA_ARGS__);     \
            throw ::tsmv::Err{TSMV_EINVAL};     \
        }                                       \
    } while (0)

// ------------------------------------------------------------------ tile traits
template <int NT> struct Tr;
template <> struct Tr<16> { using word_t = uint16_t; using idx_t = uint8_t;  using cs_t = uint8_t;  static constexpr int LOG = 4; };
template <> struct Tr<32> { using word_t = uint32_t; using idx_t = uint16_t; using cs_t = uint16_t; static constexpr int LOG = 5; };
template <> struct Tr<64> { using word_t = unsigned long long; using idx_t = uint16_t; using cs_t = uint16_t; static constexpr int LOG = 6; };

// Per-tile descriptor read once a tile's mask intersects x (one 16-byte load).
struct __align__(16) TileDesc {
    long long off;  // first in-tile nonzero
    int trow;       // tile row I
    int nnz;        // nonzeros in the tile
};

// nt = 16 tile record of the flat SpMSpV kernel (spmspv_flat.cu): one 64-byte
// DRAM access per hit tile.  b = the tile's 16 index bytes ((c << 4) | r,
// column-major; padding 0xff) when nnz <= 16, else its 16 column starts; v = the
// tile's values inline when they fit (nnz <= 4 fp64 / 8 fp32), else unused.
struct __align__(64) TileRec64 {
    uint32_t off;   // first in-tile nonzero in idx / val (dense_nnz < 2^32 required)
    int32_t trow;   // tile row I, or ~hot index (as TileDesc::trow)
    uint32_t nnz;
    uint32_t pad;
    uint4 b;
    uint4 v[2];
};
// Per-column record of the flat kernel: side-matrix start of column j and the
// tile range of its tile column J = j / 16 (replicated over the 16 columns), so
// that one x entry costs one 16-byte access (+ the next column's sbeg).
struct __align__(16) ColInfo {
    long long sbeg;            // side nonzeros of column j are [sbeg, next.sbeg)
    unsigned long long tinfo;  // (first tile of J << 24) | number of tiles of J
};

inline int log2_nt(int nt) { return nt == 16 ? 4 : nt == 32 ? 5 : 6; }
inline int idx_bytes(int nt) { return nt == 16 ? 1 : 2; }
inline int word_bytes(int nt) { return nt / 8; }

// ------------------------------------------------------------------ device memory
// Owning device buffer (RAII: freed on scope exit, move-only), so that builder
// temporaries can never outlive the call that made them.
struct DevBuf {
    void *p = nullptr;
    size_t bytes = 0;
    DevBuf() = default;
    DevBuf(const DevBuf &) = delete;
    DevBuf &operator=(const DevBuf &) = delete;
    DevBuf(DevBuf &&o) noexcept : p(o.p), bytes(o.bytes) {
        o.p = nullptr;
        o.bytes = 0;
    }
    DevBuf &operator=(DevBuf &&o) noexcept {
        if (this != &o) {
            release();
            p = o.p;
            bytes = o.bytes;
            o.p = nullptr;
            o.bytes = 0;
        }
        return *this;
    }
    ~DevBuf() { release(); }
    void alloc(size_t b) {
        release();
        if (b == 0) b = 16;
        TSMV_CUDA(cudaMalloc(&p, b));
        bytes = b;
    }
    void ensure(size_t b) {
        if (b > bytes) alloc(b);
    }
    void release() {
        if (p) cudaFree(p);
        p = nullptr;
        bytes = 0;
    }
    template <class T> T *as() const { return static_cast<T *>(p); }
};

// One tile-CSC ("TileSet") built from a set of (row, col[, val]) entries of a
// dimR x dimC matrix.  For A itself (push / SpMSpV) rows are A's rows; for the
// pull structure of a directed graph it is built from A^T.
struct TileSet {
    int64_t dimR = 0, dimC = 0, nTR = 0, nTC = 0;
    int64_t n_tiles_all = 0;  // non-empty tiles before extraction
    int64_t T = 0;            // tiles kept (dense)
    int64_t dense_nnz = 0, side_nnz = 0;
    DevBuf ptr;      // int64[nTC+1]: tiles of tile column J are [ptr[J], ptr[J+1])
    DevBuf trow;     // int32[T]: tile row I of each tile
    DevBuf tgrp;     // int32[T]: tile column J of each tile (group id)
    DevBuf mask;     // word_t[T]: column-occupancy mask (bit c = column c non-empty)
    DevBuf off;      // int64[T+1]: first in-tile nonzero of each tile
    DevBuf idx;      // idx_t[dense_nnz]: (c << LOG) | r, column-major inside a tile
    DevBuf val;      // double/float[dense_nnz] (absent for pattern)
    DevBuf planes;   // word_t[NT][T]: plane c holds column word c of every tile (bit r = row r)
    DevBuf pmask;    // u64[nTC]: bit c = plane c non-empty in some tile of group J (pull: rows with tile in-edges)
    DevBuf smask;    // u32[ceil(dimC/32)]: bit = side column non-empty (pull: rows with side in-edges)
    DevBuf desc;     // TileDesc[T]
    DevBuf cstart;   // cs_t[T][NT]: start of column c inside the tile's nonzeros (column-major)
    DevBuf rec;      // TileRec64[T] (nt = 16 only): descriptor + inline indices / column starts / values
    DevBuf colinfo;  // ColInfo[dimC + 1] (nt = 16 only)
    DevBuf sptr;     // int64[dimC+1]: side matrix (very sparse tiles), CSC
    DevBuf srow;     // int32[side_nnz]
    DevBuf sval;     // double/float[side_nnz]
    bool has_vals = false, has_planes = false, has_list = false;
    // Hot-row encoding (SpMSpV privatisation): rows of "hot" tile rows
    // are stored as ~(hot_idx*NT + r) in srow and as ~hot_idx in TileDesc::trow;
    // hot_list[hot_idx] = tile row.  decode_row() restores the row id.
    const int32_t *hot_list = nullptr;
    size_t bytes() const {
        return ptr.bytes + trow.bytes + tgrp.bytes + mask.bytes + off.bytes + idx.bytes + val.bytes +
               planes.bytes + pmask.bytes + smask.bytes + sptr.bytes + srow.bytes + sval.bytes + desc.bytes + cstart.bytes + rec.bytes + colinfo.bytes;
    }
    void release() {
        for (DevBuf *b : {&ptr, &trow, &tgrp, &mask, &off, &idx, &val, &planes, &pmask, &smask, &sptr, &srow, &sval, &desc, &cstart, &rec, &colinfo})
            b->release();
    }
};

// Device counters shared by the kernels of one call (one cache line each group).
struct Counters {
    // x / frontier scan results
    long long nLt, Wt, nLs, Ws;    // segment list size, tile work, side list size, side work
    long long nCt, nCs;            // chunk counts
    long long fsize, mf, din;      // BFS: |F|, sum outdeg(F), sum indeg(new owned)
    long long y_nnz;
    int err;                       // 1 = x not strictly ascending / out of range
    int pad0;
    unsigned int bid_scan;         // dynamic block-id counters (reset by the next kernel)
    unsigned int bid_compact;
    unsigned int chunk_next;       // work-queue head of the expand kernel
    unsigned int pad1;
    long long reached, edges;      // BFS totals
    long long hit_tiles, hit_nnz, tile_macs;  // expand-kernel accounting (tiles with mask hit,
                                              // their nonzeros, useful multiplies in tiles)
    unsigned long long bar;        // grid-barrier arrival counter (monotonic)
    unsigned long long resv_t;     // flat SpMSpV list reservation: (entries << 40) | tile work
    unsigned long long resv_s;     // (entries << 37) | side work; reset at the end of each call
    unsigned long long nhits;      // flat SpMSpV: hit tiles appended in phase B1
    unsigned long long bfs_bars;   // fused BFS: grid barriers the last launch passed
    unsigned int fscan_ticket;     // stats-only frontier scan: blocks done (last one publishes)
    unsigned int pad2;
};

template <int K> struct LBDesc {
    long long agg[K];
    long long inc[K];
    unsigned int status;  // (epoch << 2) | flag ; flag 1 = aggregate, 2 = inclusive prefix
    unsigned int pad;
};

// Per-call list workspace (capacity grows on demand).
struct Lists {
    int64_t cap_seg = 0, cap_ent = 0, cap_ct = 0, cap_cs = 0, cap_blk = 0;
    DevBuf Lt_seg, Lt_mask, Lt_first, Lt_tbeg, Lt_wpre;  // per non-empty segment with tiles
    DevBuf Ls_beg, Ls_wpre, Ls_x, Ls_col;                // per x entry / vertex with side work
    DevBuf Ct, Cs;                                        // chunk -> first list index
    DevBuf xv;                                            // x values as double
    DevBuf desc_scan;                                     // LBDesc<4>[blocks]
    size_t bytes() const {
        return Lt_seg.bytes + Lt_mask.bytes + Lt_first.bytes + Lt_tbeg.bytes + Lt_wpre.bytes +
               Ls_beg.bytes + Ls_wpre.bytes + Ls_x.bytes + Ls_col.bytes + Ct.bytes + Cs.bytes +
               xv.bytes + desc_scan.bytes;
    }
    void release() {
        for (DevBuf *b : {&Lt_seg, &Lt_mask, &Lt_first, &Lt_tbeg, &Lt_wpre, &Ls_beg, &Ls_wpre, &Ls_x,
                          &Ls_col, &Ct, &Cs, &xv, &desc_scan})
            b->release();
    }
};

// Per-call lists of the flat SpMSpV kernel (capacity grows on demand).
struct FlatLists {
    int64_t cap_ent = 0;
    DevBuf t_beg, t_wpre, t_xm, t_J;  // per x segment with tiles: first tile, work prefix, x bits, J
    DevBuf t_xv;                      // double[16] per segment with tiles: its x values by column
    DevBuf s_beg, s_wpre, s_x;        // per x entry with side work: first side nonzero, prefix, x_j
    DevBuf Ct, Cs;                    // chunk -> first list entry
    DevBuf hits;                      // uint4 {tile, hit columns, segment slot, 0} per hit tile
    DevBuf pcnt;                      // u32[2][MAXG * KP]: touched rows per bitmap piece (2 buffers)
    size_t bytes() const {
        return t_beg.bytes + t_wpre.bytes + t_xm.bytes + t_J.bytes + t_xv.bytes + s_beg.bytes + s_wpre.bytes + s_x.bytes +
               Ct.bytes + Cs.bytes + hits.bytes;
    }
    void release() {
        for (DevBuf *b : {&t_beg, &t_wpre, &t_xm, &t_J, &t_xv, &s_beg, &s_wpre, &s_x, &Ct, &Cs, &hits, &pcnt}) b->release();
    }
};
struct FlatListsView {
    long long *t_beg, *t_wpre;
    unsigned *t_xm;
    int *t_J;
    double *t_xv;
    long long *s_beg, *s_wpre;
    double *s_x;
    int *Ct, *Cs;
    uint4 *hits;
    long long *pcnt;
    double *xd;
};

#ifndef TSMV_HOT_SLOTS
#define TSMV_HOT_SLOTS 2048
#endif
constexpr int HOT_SLOTS = TSMV_HOT_SLOTS;  // privatised rows per CTA (smem fp64 + bits)
constexpr int CHUNK_LOG = 7;               // 128 work items per warp-chunk
constexpr int CHUNK = 1 << CHUNK_LOG;
constexpr int SCAN_BLOCK = 256;

}  // namespace tsmv

struct tsmv_ctx {
    int device = 0;
    tsmv_options opt{};
    tsmv_dtype dtype = TSMV_F64;
    int nt = 16, lognt = 4;
    int64_t m = 0, n = 0, nnz = 0, row_begin = 0;
    int64_t nTR = 0, nTC = 0;
    int sm_count = 148;
    int expand_blocks = 0;     // persistent grid of the expand kernels
    bool symmetric = false;
    bool bfs_built = false;
    double build_ms = 0;
    std::vector<int64_t> row_splits;

    tsmv::TileSet P;           // tile-CSC of A (SpMSpV + push kernels)
    tsmv::TileSet Qown;        // tile-CSC of A^T (pull / Push-CSR) when A is not symmetric
    tsmv::TileSet *Q = nullptr;

    tsmv::DevBuf hot_list;     // int32[n_hot]: tile rows privatised in the SpMSpV kernel
    int n_hot = 0;
    tsmv::DevBuf outdeg;       // int32[n]: nnz of column v (local rows)
    tsmv::DevBuf indeg;        // int32[m]: nnz of row v

    // SpMSpV workspaces (clear-on-read)
    tsmv::DevBuf acc;          // double[m] (or ordered keys for MIN)
    tsmv::DevBuf xdense;       // double[n]: x_j scattered by column (only x's columns are ever read)
    tsmv::DevBuf acct;         // long long[expand_blocks][4]: per-block byte-accounting counters
    tsmv::DevBuf rowbits;      // (unused; the bitmap lives in `acc`, see rowbits_p)
    uint32_t *rowbits_p = nullptr;  // uint32[ceil(m/32)] touched rows, inside the acc allocation
    size_t persist_bytes = 0;  // L2 persisting window over acc (+ bitmap); 0 = none
    float persist_ratio = 0.f;
    tsmv::DevBuf desc_compact; // LBDesc<1>[blocks]
    tsmv::Lists L;
    tsmv::FlatLists FL;
    tsmv::DevBuf counters;     // Counters
    tsmv::Counters *hcnt = nullptr;  // mapped pinned mirror written by kernels
    tsmv::Counters *hcnt_dev = nullptr;
    unsigned int epoch = 0;

    // host staging
    tsmv::DevBuf stage_x_idx, stage_x_val, stage_y_idx, stage_y_val, stage_levels;
    tsmv::DevBuf sort_x_idx, sort_x_val, sort_tmp;  // x sorted by tsmv_spmspv when not ascending (R21)

    // BFS state
    tsmv::DevBuf V, F0, F1;    // uint32[ceil(n/64)*2] visited, frontier ping-pong
    tsmv::DevBuf desc_bfs;     // LBDesc<8>[ceil(nTC/256)+1]
    tsmv::DevBuf splits_dev;   // int64[nranks+1]
    int fcur = 0;
    int32_t *levels_dev = nullptr;
    int bfs_level = 0;
    long long m_u_local = 0;
    long long cur_fsize = 0, cur_mf = 0;

    cudaEvent_t ev0 = nullptr, ev1 = nullptr;
    cudaStream_t aux_stream = nullptr;          // second stream of the dense pull level (bfs.cu)
    cudaEvent_t ev_fork = nullptr, ev_join = nullptr;
    // optional per-phase timing of tsmv_spmspv* (tsmv_set_timing): block 0 of the
    // fused kernel stamps %globaltimer at its phase boundaries into a ring
    bool timing = false;
    tsmv::DevBuf tring;            // unsigned long long[TRING][8]
    long long tcalls = 0;          // timed calls since tsmv_set_timing
    unsigned long long bar_base = 0;  // value of Counters::bar at the next launch
    int fused_blocks = 0, fused_threads = 1024;
    bool use_flat = false;         // SpMSpV through the flat kernel (nt = 16), decided at create
    bool use_rows = false;         // row-driven kernel (Alg 4, spmspv_rows.cu) available (nt = 16)
    int rows_G = 0;                // CTAs of the row-driven kernel
    tsmv::DevBuf rt_row, rt_J, rt_id, rt_mask;  // dense tiles of P in row-major order
    tsmv::DevBuf rt_wstart;        // int64[rows_G * 32 + 1]: per-warp tile ranges (row-tile aligned)
    tsmv::DevBuf xbits;            // u32[n/32 + 1]: x bitmap of the row-driven kernel (zero between calls)
    int flat_blocks = 0;           // CTAs of the flat SpMSpV kernel (1024 threads, 1 per SM)
    long long flat_calls = 0;      // flat SpMSpV launches so far (piece-count buffer parity)
    int last_blocks = 0;           // CTAs of the last SpMSpV launch (partials / acct rows)
    tsmv::DevBuf partials;         // long long[fused_blocks][8]
    // bucketed flat SpMSpV (propagation blocking, spmspv_flat.cu), set up on first use
    int pb_state = 0;              // 0 = not yet, 1 = ready, -1 = unavailable (too many buckets)
    int pb_bl = 0, pb_nb = 0, pb_cap = 0;
    long long pb_calls = 0;        // bucketed launches so far (counter parity, look-back epoch)
    tsmv::DevBuf pb_rs;            // int64[NB + 1]: staging region of bucket q (nonzeros of its rows)
    tsmv::DevBuf pb_row, pb_val;   // u32[nnz], u64[nnz]: staged products / compacted output rows
    tsmv::DevBuf pb_cnt;           // u32[2][NB]: staged products per bucket, double-buffered by call parity
    tsmv::DevBuf pb_agg;           // u64[2][MAXG]: look-back aggregates, contributed list lengths
    tsmv::DevBuf pb_hp;            // u64[MAXG][hot slots]: per-CTA hot-row partials
    tsmv::DevBuf pb_hr;            // u64[hot slots] reduced values + u32[hot slots] their epochs
    tsmv::DevBuf pb_hs, pb_hso;    // int32: hot slots by bucket, and their offsets [NB + 1]
    long long last_x_nnz = 0;
    int32_t *hy_idx = nullptr;     // mapped pinned host y of the synchronous call being enqueued (or null)
    void *hy_val = nullptr;
    bool hy_by_kernel = false;     // the flat kernel's phase C took the host copy over
    int bfs_blocks = 0;            // CTAs of the fused BFS kernel
    long long bfs_last_levels = 0;
    int bfs_stop_kind = 0;         // why the last persistent BFS launch stopped (1 pull, 2 bulk push)
    tsmv::DevBuf bfs_dirs, bfs_front;  // per-level direction / frontier size (device)
    tsmv::DevBuf bfs_tlv;              // u64[TSMV_MAX_LEVELS + 1]: %globaltimer at each level's decision
    // list-driven push levels of the fused BFS kernel
    tsmv::DevBuf lwork;        // int32[n]: push work of vertex u = tiles of its tile column + its side nonzeros
    tsmv::DevBuf bq0, bq1;     // int32[n]: frontier vertex lists, ping-pong by level parity
    tsmv::DevBuf lslots;       // long long[3][4]: {|F|, m_f, sum indeg, max lwork} of levels L, L+1, L+2
    // multi-source BFS (msbfs.cu), allocated on first use
    tsmv::DevBuf ms_V, ms_F0, ms_F1, ms_N;  // u64[m]: one bit per source
    tsmv::DevBuf ms_seg0, ms_seg1;          // u32: 1 bit per 16-vertex segment holding frontier vertices
    tsmv::DevBuf ms_src, ms_out;
    tsmv::DevBuf ms_rowneed;                // u16 per row tile: rows still missing some source
    tsmv::DevBuf mu_dev;                    // distributed BFS: m_u of this rank on the device
    tsmv::DevBuf dstats;                    // distributed BFS: u64[4] statistics shares of the next frontier
    tsmv::DevBuf dstats_all;                // distributed BFS: u64[nranks][4] gathered shares (comm path)
    tsmv::DevBuf b2d_bsum, b2d_boff, b2d_total, b2d_temp;  // 2D BFS bitmap -> list scratch (bfs2d.cu)
    bool bfs_block2d = false;               // build_bfs = 2: a 2D-partition block (bfs2d only)
    tsmv::DevBuf par_chunks;                // BFS parents: (vertex << 24 | chunk) of heavy side rows
    long long par_nchunks = 0;
    void *trace = nullptr;         // tsmv_set_trace (device, u64[tsmv_trace_words])
    // distributed context with its own NCCL communicator (comm.cu)
    void *nccl_comm = nullptr;     // ncclComm_t
    tsmv::DevBuf outdeg_g;         // int32[n]: global column counts (all ranks' blocks)
    tsmv::DevBuf indeg_g;          // int32[n]: global row counts
    long long nnz_global = 0;
    tsmv::DevBuf kcounts;          // int64[nranks + 1]: x counts of the ranks (SpMSpV exchange)
    tsmv::DevBuf xg_idx, xg_val;   // the gathered global x
};

namespace tsmv {
// side-matrix / descriptor row decode (hot-row encoding, see TileSet::hot_list)
template <int NT> __host__ __device__ __forceinline__ long long decode_row(long long v, const int32_t *hot_list) {
    if (v >= 0) return v;
    const long long s = ~v;
    return (long long)hot_list[s / NT] * NT + (s % NT);
}
// builder.cu
void build_tileset(tsmv_ctx *c, TileSet &S, const int32_t *rows, const int32_t *cols, const void *vals,
                   int64_t nnz, int64_t dimR, int64_t dimC, bool want_vals, bool want_planes,
                   cudaStream_t st, const int32_t *hot_map = nullptr);
void choose_hot_rows(tsmv_ctx *c, cudaStream_t st, DevBuf &hot_map);
bool same_pattern_transposed(tsmv_ctx *c, const int32_t *rows, const int32_t *cols, int64_t nnz,
                             cudaStream_t st);
void prepare_csr(tsmv_ctx *c, const int64_t *row_ptr, const int32_t *col_idx, int32_t *rows, cudaStream_t st);
// spmspv.cu
void ensure_lists(tsmv_ctx *c, int64_t k);
// spmspv_flat.cu
bool flat_supported(const tsmv_ctx *c);
void flat_init(tsmv_ctx *c, cudaStream_t st);
void build_rec64(tsmv_ctx *c, TileSet &S, cudaStream_t st);
int flat_occupancy(int dtype);
void enqueue_spmspv_flat(tsmv_ctx *c, int sr, long long k, const int32_t *xi, const void *xv, long long ycap,
                         int32_t *yi, void *yv, long long *ynnz_dev, cudaStream_t st);
void ensure_flat_lists(tsmv_ctx *c, int64_t k);
// spmspv_rows.cu
void build_row_tiles(tsmv_ctx *c, cudaStream_t st);
void enqueue_spmspv_rows(tsmv_ctx *c, int sr, long long k, const int32_t *xi, const void *xv, long long ycap,
                         int32_t *yi, void *yv, long long *ynnz_dev, cudaStream_t st);
bool use_rows_kernel(const tsmv_ctx *c, long long k);
// bfs_fused.cu
int bfs_fused_occupancy(int nt);
long long bfs_wide_cap(const tsmv_ctx *c, bool resume);  // m_u above which a wide pull level leaves the fused kernel
void bfs_list_init(tsmv_ctx *c, cudaStream_t st);
void heavy_side_chunks(tsmv_ctx *c, cudaStream_t st);  // bfs.cu: chunks of side rows > 32 entries
bool bfs_fused_launch(tsmv_ctx *c, long long source, cudaStream_t st, bool resume, long long level0, uint32_t *Fa,
                      uint32_t *Fb, long long mu, long long reached, long long edges, bool stop_on_pull,
                      long long max_levels, long long &level_out, long long &mu_out, long long &reached_out,
                      long long &edges_out, int &cur_out, long long fprev0, long long &fprev_out);
// comm.cu
bool has_comm(const tsmv_ctx *c);
void comm_init(tsmv_ctx *c, const void *unique_id, cudaStream_t st);
void comm_destroy(tsmv_ctx *c);
void comm_exchange_frontier(tsmv_ctx *c, uint32_t *F, uint32_t *V, long long nwords, const void *stats_send,
                            void *stats_all, cudaStream_t st);
long long comm_gather_x(tsmv_ctx *c, long long k_local, const int32_t *x_idx, const void *x_val, size_t vb,
                        const int32_t **xi_out, const void **xv_out, cudaStream_t st);
// bfs.cu
int choose_dir(const tsmv_options &o, long long n, long long fsize, long long mf, long long mu, long long fprev);
// reading R9': alpha of a level from the frontier's growth
__host__ __device__ __forceinline__ double burst_alpha(double alpha, double alpha_burst, double growth, long long f,
                                                       long long fprev) {
    return (alpha_burst > 0 && fprev > 0 && (double)f >= growth * (double)fprev) ? alpha_burst : alpha;
}
// pointer classification
bool is_device_ptr(const void *p);
// device address of page-locked, mapped host memory (cudaHostAlloc / torch
// pin_memory under UVA), or NULL for pageable / device memory
void *mapped_device_ptr(const void *p);
}  // namespace tsmv
