// api.cu -- C-ABI entry points of libtsmv.so other than the hot calls
// (tsmv_spmspv in spmspv.cu, tsmv_bfs* in bfs.cu): options, create/destroy,
// census, export (round-trip tests), errors.
#include "common.cuh"
#include <algorithm>
#include <cstdarg>
#include <map>
#include <mutex>
#include <tuple>

namespace tsmv {

static thread_local char g_err[1024] = "";

void set_error(const char *fmt, ...) {
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(g_err, sizeof(g_err), fmt, ap);
    va_end(ap);
}

bool is_device_ptr(const void *p) {
    if (!p) return false;
    cudaPointerAttributes a;
    cudaError_t e = cudaPointerGetAttributes(&a, p);
    if (e != cudaSuccess) {
        cudaGetLastError();
        return false;
    }
    return a.type == cudaMemoryTypeDevice || a.type == cudaMemoryTypeManaged;
}

void *mapped_device_ptr(const void *p) {
    if (!p) return nullptr;
    cudaPointerAttributes a;
    cudaError_t e = cudaPointerGetAttributes(&a, p);
    if (e != cudaSuccess) {
        cudaGetLastError();
        return nullptr;
    }
    return a.type == cudaMemoryTypeHost ? a.devicePointer : nullptr;
}

}  // namespace tsmv

using namespace tsmv;

// defined in spmspv.cu / bfs.cu (occupancy of the persistent expand kernels)
namespace tsmv {
int expand_occupancy(int nt, int dtype);
int fused_occupancy(int nt, int dtype);

// L2 residency of the SpMSpV workspace (accumulator + touched bitmap, all zero
// between calls): a persisting access-policy window on the SpMSpV launches keeps
// its lines in L2 across calls, so the first RED to a row does not fetch a zero
// sector from HBM.  Device-wide set-aside (cudaLimitPersistingL2CacheSize) is
// raised to the window size if the device allows it.  Opt-in since r2 session 5
// (TSMV_PERSIST=1): measured on B200 it left the DRAM traffic of the SpMSpV call at
// T unchanged (42.7 MB per launch either way) while the device-wide set-aside cost
// the other workloads L2 (R-MAT s26 TileBFS 682 -> 844 GTEPS and s26 SpMSpV 25 ->
// 36 GFLOP/s without it), and it let the workspace survive the bench's L2 flush.
// The device-wide set-aside is raised only while a context that uses it lives:
// the first such context records the limit it found, the last one restores it
// (and returns the persisting lines to normal), so the library leaves no L2
// policy behind once every context is destroyed.
static std::mutex g_persist_mu;
static std::map<int, std::pair<int, size_t>> g_persist;  // device -> (contexts, limit found)

static void setup_persistence(tsmv_ctx *c) {
    c->persist_bytes = 0;
    c->persist_ratio = 0.f;
    if (!getenv("TSMV_PERSIST")) return;
    int max_persist = 0, max_win = 0;
    if (cudaDeviceGetAttribute(&max_persist, cudaDevAttrMaxPersistingL2CacheSize, c->device) != cudaSuccess ||
        cudaDeviceGetAttribute(&max_win, cudaDevAttrMaxAccessPolicyWindowSize, c->device) != cudaSuccess) {
        cudaGetLastError();
        return;
    }
    if (max_persist <= 0 || max_win <= 0) return;
    const size_t want = std::min<size_t>(c->acc.bytes, (size_t)max_win);
    std::lock_guard<std::mutex> lk(g_persist_mu);
    size_t cur = 0;
    cudaDeviceGetLimit(&cur, cudaLimitPersistingL2CacheSize);
    const size_t setp = std::max(cur, std::min(want, (size_t)max_persist));
    auto it = g_persist.find(c->device);
    const size_t found = it == g_persist.end() ? cur : it->second.second;
    if (setp > cur && cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, setp) != cudaSuccess) {
        cudaGetLastError();
        return;
    }
    g_persist[c->device] = {it == g_persist.end() ? 1 : it->second.first + 1, found};
    c->persist_bytes = want;
    c->persist_ratio = (float)std::min(1.0, (double)setp / (double)want);
}

static void release_persistence(tsmv_ctx *c) {
    if (!c->persist_bytes) return;
    std::lock_guard<std::mutex> lk(g_persist_mu);
    auto it = g_persist.find(c->device);
    if (it == g_persist.end()) return;
    if (--it->second.first == 0) {
        cudaCtxResetPersistingL2Cache();
        cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, it->second.second);
        cudaGetLastError();
        g_persist.erase(it);
    }
    c->persist_bytes = 0;
}
}

extern "C" tsmv_status tsmv_default_options(tsmv_options *o) {
    if (!o) return TSMV_EINVAL;
    memset(o, 0, sizeof(*o));
    o->device = 0;
    o->tile_dim = 16;
    o->sparse_tile_max_nnz = 2;
    o->build_bfs = -1;  // auto: square and single rank
    // direction rule R9 with the thresholds measured on B200 (DESIGN.md §6,
    // profiles/r02_bfs_knobs.txt); the paper's 0.01 and Beamer's 14 stay selectable
    o->push_csr_density = 0.05;
    o->pull_alpha = 2.0;
    o->force_dir = TSMV_DIR_AUTO;
    o->row_driven_density = 0.05;  // measured crossover
    o->pull_alpha_burst = 14.0;    // reading R9': Beamer's alpha on explosive levels
    o->burst_growth = 4.0;
    o->rank = 0;
    o->nranks = 1;
    o->row_begin = 0;
    o->row_splits = nullptr;
    return TSMV_OK;
}

extern "C" const char *tsmv_last_error(void) { return g_err; }
extern "C" int32_t tsmv_version(void) { return TSMV_VERSION; }

static void destroy_impl(tsmv_ctx *c) {
    if (!c) return;
    cudaSetDevice(c->device);
    cudaDeviceSynchronize();
    comm_destroy(c);
    release_persistence(c);
    c->P.release();
    c->Qown.release();
    for (DevBuf *b : {&c->outdeg, &c->indeg, &c->acc, &c->rowbits, &c->desc_compact, &c->counters, &c->stage_x_idx,
                      &c->stage_x_val, &c->stage_y_idx, &c->stage_y_val, &c->stage_levels, &c->V, &c->F0, &c->F1,
                      &c->desc_bfs, &c->splits_dev, &c->xdense, &c->acct, &c->tring, &c->partials, &c->hot_list, &c->bfs_dirs, &c->bfs_front, &c->bfs_tlv, &c->lwork, &c->bq0,
                      &c->bq1, &c->lslots})
        b->release();
    c->L.release();
    c->FL.release();
    if (c->hcnt) cudaFreeHost(c->hcnt);
    if (c->ev0) cudaEventDestroy(c->ev0);
    if (c->ev_fork) cudaEventDestroy(c->ev_fork);
    if (c->ev_join) cudaEventDestroy(c->ev_join);
    if (c->aux_stream) cudaStreamDestroy(c->aux_stream);
    if (c->ev1) cudaEventDestroy(c->ev1);
    delete c;
}

extern "C" tsmv_status tsmv_create(tsmv_ctx **out, int64_t nrows, int64_t ncols, const int64_t *row_ptr,
                                   const int32_t *col_idx, const void *values, tsmv_dtype dtype,
                                   const tsmv_options *opt) {
    tsmv_ctx *c = nullptr;
    cudaStream_t st = nullptr;
    try {
        TSMV_REQUIRE(out != nullptr, "tsmv_create: NULL out");
        *out = nullptr;
        TSMV_REQUIRE(nrows >= 0 && ncols >= 1 && ncols < (1ll << 31) && nrows < (1ll << 31),
                     "tsmv_create: bad sizes %lld x %lld", (long long)nrows, (long long)ncols);
        TSMV_REQUIRE(row_ptr != nullptr, "tsmv_create: NULL row_ptr");
        TSMV_REQUIRE(dtype >= TSMV_F64 && dtype <= TSMV_PATTERN, "tsmv_create: bad dtype");
        TSMV_REQUIRE((dtype == TSMV_PATTERN) == (values == nullptr),
                     "tsmv_create: values must be NULL iff dtype == TSMV_PATTERN");
        c = new tsmv_ctx();
        if (opt) c->opt = *opt;
        else tsmv_default_options(&c->opt);
        const tsmv_options &o = c->opt;
        TSMV_REQUIRE(o.tile_dim == 16 || o.tile_dim == 32 || o.tile_dim == 64, "tsmv_create: tile_dim must be 16|32|64");
        TSMV_REQUIRE(o.sparse_tile_max_nnz >= 0, "tsmv_create: sparse_tile_max_nnz < 0");
        TSMV_REQUIRE(o.nranks >= 1 && o.rank >= 0 && o.rank < o.nranks, "tsmv_create: bad rank/nranks");
        TSMV_REQUIRE(o.pull_alpha > 0 && o.push_csr_density >= 0, "tsmv_create: bad direction thresholds");
        TSMV_REQUIRE(o.force_dir >= 0 && o.force_dir <= 3, "tsmv_create: bad force_dir");
        c->device = o.device;
        c->dtype = dtype;
        c->nt = o.tile_dim;
        c->lognt = log2_nt(c->nt);
        c->m = nrows;
        c->n = ncols;
        if (o.nranks == 1 && o.nccl_unique_id) {
            // a one-rank communicator (tests the collective path on one GPU)
            TSMV_REQUIRE(o.row_begin == 0, "tsmv_create: row_begin must be 0 when nranks == 1");
            c->row_splits = {0, nrows};
            c->row_begin = 0;
        } else if (o.nranks > 1) {
            TSMV_REQUIRE(o.row_splits != nullptr, "tsmv_create: nranks > 1 needs row_splits");
            c->row_splits.assign(o.row_splits, o.row_splits + o.nranks + 1);
            for (int p = 0; p <= o.nranks; ++p) {
                TSMV_REQUIRE(p == 0 || c->row_splits[p] >= c->row_splits[p - 1], "tsmv_create: row_splits not monotone");
                TSMV_REQUIRE(p == o.nranks || c->row_splits[p] % 64 == 0,
                             "tsmv_create: row_splits must be multiples of 64");
            }
            TSMV_REQUIRE(c->row_splits[0] == 0 && c->row_splits[o.nranks] == ncols,
                         "tsmv_create: row_splits must cover [0, ncols) (square partitioned A)");
            TSMV_REQUIRE(c->row_splits[o.rank + 1] - c->row_splits[o.rank] == nrows,
                         "tsmv_create: nrows != owned rows of this rank");
            c->row_begin = c->row_splits[o.rank];
        } else {
            TSMV_REQUIRE(o.row_begin == 0, "tsmv_create: row_begin must be 0 when nranks == 1");
            c->row_begin = 0;
        }
        bool square_global = (o.nranks == 1) ? (nrows == ncols) : true;
        const bool block2d = o.build_bfs == 2;
        TSMV_REQUIRE(!block2d || o.nranks == 1, "tsmv_create: build_bfs = 2 (2D block) needs nranks == 1");
        bool want_bfs = o.build_bfs < 0 ? square_global : o.build_bfs != 0;
        TSMV_REQUIRE(!want_bfs || square_global || block2d, "tsmv_create: build_bfs needs a square matrix");
        c->opt.build_bfs = block2d ? 2 : want_bfs ? 1 : 0;
        c->bfs_block2d = block2d;

        TSMV_CUDA(cudaSetDevice(c->device));
        // device inputs may still be in flight on the caller's streams
        TSMV_CUDA(cudaDeviceSynchronize());
        cudaDeviceProp prop;
        TSMV_CUDA(cudaGetDeviceProperties(&prop, c->device));
        c->sm_count = prop.multiProcessorCount;
        TSMV_CUDA(cudaStreamCreateWithFlags(&st, cudaStreamNonBlocking));
        TSMV_CUDA(cudaEventCreate(&c->ev0));
        TSMV_CUDA(cudaEventCreate(&c->ev1));
        TSMV_CUDA(cudaStreamCreateWithFlags(&c->aux_stream, cudaStreamNonBlocking));
        TSMV_CUDA(cudaEventCreateWithFlags(&c->ev_fork, cudaEventDisableTiming));
        TSMV_CUDA(cudaEventCreateWithFlags(&c->ev_join, cudaEventDisableTiming));
        TSMV_CUDA(cudaEventRecord(c->ev0, st));

        // --- inputs on device
        DevBuf d_rp, d_ci, d_val, d_rows;
        const int64_t *rp = row_ptr;
        int64_t nnz = 0;
        if (is_device_ptr(row_ptr)) {
            TSMV_CUDA(cudaMemcpy(&nnz, row_ptr + nrows, 8, cudaMemcpyDeviceToHost));
        } else {
            nnz = row_ptr[nrows];
            d_rp.alloc((nrows + 1) * 8);
            TSMV_CUDA(cudaMemcpyAsync(d_rp.p, row_ptr, (nrows + 1) * 8, cudaMemcpyHostToDevice, st));
            rp = d_rp.as<int64_t>();
        }
        TSMV_REQUIRE(nnz >= 0, "tsmv_create: negative nnz");
        TSMV_REQUIRE(nnz == 0 || col_idx != nullptr, "tsmv_create: NULL col_idx");
        c->nnz = nnz;
        const int32_t *ci = col_idx;
        if (nnz && !is_device_ptr(col_idx)) {
            d_ci.alloc(nnz * 4);
            TSMV_CUDA(cudaMemcpyAsync(d_ci.p, col_idx, nnz * 4, cudaMemcpyHostToDevice, st));
            ci = d_ci.as<int32_t>();
        }
        const size_t vb = dtype == TSMV_F32 ? 4 : 8;
        const void *vv = values;
        if (nnz && values && !is_device_ptr(values)) {
            d_val.alloc(nnz * vb);
            TSMV_CUDA(cudaMemcpyAsync(d_val.p, values, nnz * vb, cudaMemcpyHostToDevice, st));
            vv = d_val.p;
        }
        d_rows.alloc(std::max<int64_t>(nnz, 1) * 4);
        prepare_csr(c, rp, ci, d_rows.as<int32_t>(), st);

        // --- tiled structures
        DevBuf hot_map;
        // hot-row privatisation in the SpMSpV kernels: opt-in since r2 session 5
        // (TSMV_HOT=1); without the L2 persisting window it no longer paid (T: 53.2
        // -> 51.3 us without it, profiles/r02_pb_experiment.txt)
        if (getenv("TSMV_HOT")) choose_hot_rows(c, st, hot_map);
        build_tileset(c, c->P, d_rows.as<int32_t>(), ci, vv, nnz, nrows, ncols, dtype != TSMV_PATTERN, want_bfs, st,
                      c->n_hot ? hot_map.as<int32_t>() : nullptr);
        hot_map.release();
        build_rec64(c, c->P, st);
        build_row_tiles(c, st);
        c->nTR = c->P.nTR;
        c->nTC = c->P.nTC;
        if (want_bfs) {
            c->symmetric = (o.nranks == 1) && !block2d && same_pattern_transposed(c, d_rows.as<int32_t>(), ci, nnz, st);
            if (c->symmetric) {
                c->Q = &c->P;
            } else {
                // A^T: rows <- columns of A (dimR = ncols), columns <- local rows (dimC = nrows)
                build_tileset(c, c->Qown, ci, d_rows.as<int32_t>(), nullptr, nnz, ncols, nrows, false, true, st);
                c->Q = &c->Qown;
            }
            c->bfs_built = true;
        }
        d_rows.release();
        d_ci.release();
        d_val.release();
        d_rp.release();

        // --- workspaces
        // accumulator and touched-row bitmap in ONE allocation, so that a single
        // L2 access-policy window can keep both resident (setup_persistence)
        int64_t W = (nrows + 31) / 32;
        const size_t acc_b = ((size_t)std::max<int64_t>(nrows, 1) * 8 + 255) & ~(size_t)255;
        c->acc.alloc(acc_b + (size_t)std::max<int64_t>(W, 1) * 4);
        TSMV_CUDA(cudaMemsetAsync(c->acc.p, 0, c->acc.bytes, st));
        c->rowbits_p = reinterpret_cast<uint32_t *>(static_cast<char *>(c->acc.p) + acc_b);
        flat_init(c, st);
        setup_persistence(c);
        int64_t cblocks = (W + SCAN_BLOCK - 1) / SCAN_BLOCK + 1;
        c->desc_compact.alloc(cblocks * sizeof(LBDesc<1>));
        TSMV_CUDA(cudaMemsetAsync(c->desc_compact.p, 0, c->desc_compact.bytes, st));
        c->counters.alloc(sizeof(Counters));
        TSMV_CUDA(cudaMemsetAsync(c->counters.p, 0, sizeof(Counters), st));
        TSMV_CUDA(cudaHostAlloc((void **)&c->hcnt, sizeof(Counters), cudaHostAllocMapped));
        memset(c->hcnt, 0, sizeof(Counters));
        TSMV_CUDA(cudaHostGetDevicePointer((void **)&c->hcnt_dev, c->hcnt, 0));
        if (want_bfs) {
            int64_t NWpad = ((ncols + 127) / 128) * 4;  // whole 16-byte vectors (k_fscan)
            c->V.alloc(NWpad * 4);
            c->F0.alloc(NWpad * 4);
            c->F1.alloc(NWpad * 4);
            TSMV_CUDA(cudaMemsetAsync(c->F0.p, 0, c->F0.bytes, st));
            TSMV_CUDA(cudaMemsetAsync(c->F1.p, 0, c->F1.bytes, st));
            int64_t bb = (c->nTC + SCAN_BLOCK - 1) / SCAN_BLOCK + 1;
            c->desc_bfs.alloc(bb * sizeof(LBDesc<8>));
            TSMV_CUDA(cudaMemsetAsync(c->desc_bfs.p, 0, c->desc_bfs.bytes, st));
        }
        if (o.nccl_unique_id) comm_init(c, o.nccl_unique_id, st);
        if (o.nranks > 1) {
            c->splits_dev.alloc((o.nranks + 1) * 8);
            TSMV_CUDA(cudaMemcpyAsync(c->splits_dev.p, c->row_splits.data(), (o.nranks + 1) * 8,
                                      cudaMemcpyHostToDevice, st));
        }
        c->expand_blocks = c->sm_count * expand_occupancy(c->nt, (int)dtype);
        // fused SpMSpV: all CTAs co-resident (cooperative launch), up to 4 per SM
        int fo = fused_occupancy(c->nt, (int)dtype);
        TSMV_REQUIRE(fo >= 1, "tsmv_create: fused SpMSpV kernel cannot be resident (occupancy 0)");
        c->fused_blocks = c->sm_count * std::min(fo, 4);
        if (c->P.rec.p) {
            int fl = flat_occupancy((int)dtype);
            TSMV_REQUIRE(fl >= 1, "tsmv_create: flat SpMSpV kernel cannot be resident (occupancy 0)");
            c->flat_blocks = std::min(c->sm_count, 256);  // one 1024-thread CTA per SM (MAXG)
        }
        if (want_bfs && o.nranks == 1 && !block2d) {
            int bo = bfs_fused_occupancy(c->nt);
            TSMV_REQUIRE(bo >= 1, "tsmv_create: fused BFS kernel cannot be resident (occupancy 0)");
            c->bfs_blocks = c->sm_count * std::min(bo, 2);
            c->bfs_dirs.alloc(TSMV_MAX_LEVELS * 4);
            c->bfs_front.alloc(TSMV_MAX_LEVELS * 8);
            c->bfs_tlv.alloc((TSMV_MAX_LEVELS + 1) * 8);
            bfs_list_init(c, st);
        }
        c->partials.alloc((size_t)std::max({c->fused_blocks, c->bfs_blocks, c->flat_blocks}) * 8 * 8);
        TSMV_CUDA(cudaMemsetAsync(c->partials.p, 0, c->partials.bytes, st));
        c->acct.alloc((size_t)std::max({c->expand_blocks, c->fused_blocks, c->flat_blocks}) * 4 * 8);
        TSMV_CUDA(cudaMemsetAsync(c->acct.p, 0, c->acct.bytes, st));
        c->xdense.alloc(std::max<int64_t>(ncols, 1) * 8);
        TSMV_CUDA(cudaEventRecord(c->ev1, st));
        TSMV_CUDA(cudaStreamSynchronize(st));
        float ms = 0;
        TSMV_CUDA(cudaEventElapsedTime(&ms, c->ev0, c->ev1));
        c->build_ms = ms;
        cudaStreamDestroy(st);
        *out = c;
        return TSMV_OK;
    } catch (const Err &e) {
        if (st) cudaStreamDestroy(st);
        destroy_impl(c);
        return e.st;
    } catch (const std::bad_alloc &) {
        if (st) cudaStreamDestroy(st);
        destroy_impl(c);
        set_error("tsmv_create: host allocation failed");
        return TSMV_ENOMEM;
    }
}

extern "C" tsmv_status tsmv_destroy(tsmv_ctx *c) {
    destroy_impl(c);
    return TSMV_OK;
}

extern "C" tsmv_status tsmv_get_info(const tsmv_ctx *c, tsmv_info *info) {
    if (!c || !info) {
        set_error("tsmv_get_info: NULL argument");
        return TSMV_EINVAL;
    }
    memset(info, 0, sizeof(*info));
    info->nrows = c->m;
    info->ncols = c->n;
    info->nnz = c->nnz;
    info->tile_dim = c->nt;
    info->symmetric = c->symmetric ? 1 : 0;
    info->n_tiles = c->P.n_tiles_all;
    info->n_dense_tiles = c->P.T;
    info->dense_nnz = c->P.dense_nnz;
    info->side_nnz = c->P.side_nnz;
    info->bytes_spmspv = (int64_t)(c->P.bytes() - c->P.planes.bytes);
    info->bytes_bfs = (int64_t)(c->P.planes.bytes + (c->Q == &c->Qown ? c->Qown.bytes() : 0));
    info->bytes_workspace = (int64_t)(c->acc.bytes + c->rowbits.bytes + c->desc_compact.bytes + c->L.bytes() +
                                      c->V.bytes + c->F0.bytes + c->F1.bytes + c->desc_bfs.bytes +
                                      c->outdeg.bytes + c->indeg.bytes + c->pb_rs.bytes + c->pb_row.bytes +
                                      c->pb_val.bytes + c->pb_cnt.bytes + c->pb_agg.bytes +
                                      c->pb_hp.bytes + c->pb_hr.bytes + c->pb_hs.bytes + c->pb_hso.bytes);
    info->build_ms = c->build_ms;
    return TSMV_OK;
}

template <class T> static std::vector<T> d2h(const DevBuf &b, size_t count) {
    std::vector<T> h(count);
    if (count) TSMV_CUDA(cudaMemcpy(h.data(), b.p, count * sizeof(T), cudaMemcpyDeviceToHost));
    return h;
}

static tsmv_ctx *g_export_ctx = nullptr;  // set by the export entry points (single-threaded use)
static std::vector<int32_t> host_hot_list(const TileSet &S) {
    std::vector<int32_t> h;
    if (S.hot_list && g_export_ctx && g_export_ctx->n_hot) {
        h.resize(g_export_ctx->n_hot);
        TSMV_CUDA(cudaMemcpy(h.data(), S.hot_list, h.size() * 4, cudaMemcpyDeviceToHost));
    }
    return h;
}
static int64_t decode_host(int32_t v, const std::vector<int32_t> &hl, int nt) {
    if (v >= 0) return v;
    int64_t s = ~(int64_t)v;
    return (int64_t)hl[s / nt] * nt + s % nt;
}

// Host-side walk over every stored entry of a TileSet: f(row, col, dense?, value_index)
template <class F> static void walk_tileset(const TileSet &S, int nt, F f) {
    int LOG = log2_nt(nt);
    auto trow = d2h<int32_t>(S.trow, S.T);
    auto tgrp = d2h<int32_t>(S.tgrp, S.T);
    auto off = d2h<int64_t>(S.off, S.T + 1);
    std::vector<uint16_t> idx(S.dense_nnz);
    if (nt == 16) {
        auto b = d2h<uint8_t>(S.idx, S.dense_nnz);
        for (int64_t i = 0; i < S.dense_nnz; ++i) idx[i] = b[i];
    } else {
        idx = d2h<uint16_t>(S.idx, S.dense_nnz);
    }
    for (int64_t t = 0; t < S.T; ++t)
        for (int64_t p = off[t]; p < off[t + 1]; ++p) {
            int c = idx[p] >> LOG, r = idx[p] & (nt - 1);
            f((int64_t)trow[t] * nt + r, (int64_t)tgrp[t] * nt + c, true, p);
        }
    auto sptr = d2h<int64_t>(S.sptr, S.dimC + 1);
    auto srow = d2h<int32_t>(S.srow, S.side_nnz);
    std::vector<int32_t> hl = host_hot_list(S);
    for (int64_t j = 0; j < S.dimC; ++j)
        for (int64_t p = sptr[j]; p < sptr[j + 1]; ++p) f(decode_host(srow[p], hl, nt), j, false, p);
}

extern "C" tsmv_status tsmv_export_csr(tsmv_ctx *c, int64_t *row_ptr, int32_t *col_idx, void *values) {
    try {
        TSMV_REQUIRE(c && row_ptr && (c->nnz == 0 || col_idx), "tsmv_export_csr: NULL argument");
        TSMV_CUDA(cudaSetDevice(c->device));
        g_export_ctx = c;
        const TileSet &S = c->P;
        bool f32 = c->dtype == TSMV_F32;
        size_t vb = f32 ? 4 : 8;
        std::vector<uint8_t> dval, sval;
        if (values && S.has_vals) {
            dval = d2h<uint8_t>(S.val, S.dense_nnz * vb);
            sval = d2h<uint8_t>(S.sval, S.side_nnz * vb);
        }
        std::vector<std::tuple<int64_t, int64_t, double>> ent;
        ent.reserve(c->nnz);
        walk_tileset(S, c->nt, [&](int64_t r, int64_t col, bool dense, int64_t p) {
            double v = 1.0;
            if (!dval.empty() || !sval.empty()) {
                const uint8_t *src = dense ? dval.data() : sval.data();
                if (f32) {
                    float x;
                    memcpy(&x, src + p * 4, 4);
                    v = x;
                } else {
                    memcpy(&v, src + p * 8, 8);
                }
            }
            ent.emplace_back(r, col, v);
        });
        std::sort(ent.begin(), ent.end(), [](const auto &a, const auto &b) {
            return std::get<0>(a) != std::get<0>(b) ? std::get<0>(a) < std::get<0>(b) : std::get<1>(a) < std::get<1>(b);
        });
        TSMV_REQUIRE((int64_t)ent.size() == c->nnz, "tsmv_export_csr: entry count mismatch (%lld vs %lld)",
                     (long long)ent.size(), (long long)c->nnz);
        for (int64_t i = 0; i <= c->m; ++i) row_ptr[i] = 0;
        for (size_t q = 0; q < ent.size(); ++q) {
            row_ptr[std::get<0>(ent[q]) + 1] += 1;
            col_idx[q] = (int32_t)std::get<1>(ent[q]);
            if (values) {
                if (f32) ((float *)values)[q] = (float)std::get<2>(ent[q]);
                else ((double *)values)[q] = std::get<2>(ent[q]);
            }
        }
        for (int64_t i = 0; i < c->m; ++i) row_ptr[i + 1] += row_ptr[i];
        return TSMV_OK;
    } catch (const Err &e) {
        return e.st;
    }
}

extern "C" tsmv_status tsmv_export_bitmask_tiles(tsmv_ctx *c, int32_t orient, int64_t max_tiles, int64_t *tile_I,
                                                 int64_t *tile_J, uint64_t *words, int64_t *n_tiles) {
    try {
        TSMV_REQUIRE(c && tile_I && tile_J && words && n_tiles, "tsmv_export_bitmask_tiles: NULL argument");
        TSMV_REQUIRE(c->bfs_built, "tsmv_export_bitmask_tiles: no BFS structures");
        TSMV_REQUIRE(orient == 0 || orient == 1, "tsmv_export_bitmask_tiles: orient must be 0 or 1");
        TSMV_CUDA(cudaSetDevice(c->device));
        const int nt = c->nt;
        const TileSet &S = c->P;
        // dense tiles: bit planes as stored (plane c, bit r), verified against the nonzero list
        std::map<std::pair<int64_t, int64_t>, std::vector<uint64_t>> tiles;  // key (I, J), column words LSB-first
        std::vector<uint64_t> planes(S.T * nt);
        {
            size_t wb = nt / 8;
            auto raw = d2h<uint8_t>(S.planes, S.T * nt * wb);
            for (int64_t i = 0; i < S.T * nt; ++i) {
                uint64_t w = 0;
                memcpy(&w, raw.data() + i * wb, wb);
                planes[i] = w;
            }
        }
        auto trow = d2h<int32_t>(S.trow, S.T);
        auto tgrp = d2h<int32_t>(S.tgrp, S.T);
        for (int64_t t = 0; t < S.T; ++t) {
            std::vector<uint64_t> w(nt);
            for (int cc = 0; cc < nt; ++cc) w[cc] = planes[(int64_t)cc * S.T + t];
            tiles[{trow[t], tgrp[t]}] = w;
        }
        // side entries folded back into their tiles
        g_export_ctx = c;
        auto sptr = d2h<int64_t>(S.sptr, S.dimC + 1);
        auto srow = d2h<int32_t>(S.srow, S.side_nnz);
        std::vector<int32_t> hl = host_hot_list(S);
        for (int64_t j = 0; j < S.dimC; ++j)
            for (int64_t p = sptr[j]; p < sptr[j + 1]; ++p) {
                int64_t r = decode_host(srow[p], hl, nt);
                auto &w = tiles[{r / nt, j / nt}];
                if (w.empty()) w.assign(nt, 0);
                w[j % nt] |= 1ull << (r % nt);
            }
        // order + MSB-first presentation
        std::vector<std::pair<int64_t, int64_t>> keys;
        for (auto &kv : tiles) keys.push_back(kv.first);
        if (orient == 0)
            std::sort(keys.begin(), keys.end(), [](auto a, auto b) {
                return a.second != b.second ? a.second < b.second : a.first < b.first;
            });
        TSMV_REQUIRE((int64_t)keys.size() <= max_tiles, "tsmv_export_bitmask_tiles: capacity %lld < %lld",
                     (long long)max_tiles, (long long)keys.size());
        for (size_t q = 0; q < keys.size(); ++q) {
            const auto &w = tiles[keys[q]];
            tile_I[q] = keys[q].first;
            tile_J[q] = keys[q].second;
            for (int a = 0; a < nt; ++a) {
                uint64_t out = 0;
                for (int b = 0; b < nt; ++b) {
                    // orient 0: word a = column a, bit for row b; orient 1: word a = row a, bit for column b
                    bool set = orient == 0 ? ((w[a] >> b) & 1) : ((w[b] >> a) & 1);
                    if (set) out |= 1ull << (nt - 1 - b);
                }
                words[q * nt + a] = out;
            }
        }
        *n_tiles = (int64_t)keys.size();
        return TSMV_OK;
    } catch (const Err &e) {
        return e.st;
    }
}
