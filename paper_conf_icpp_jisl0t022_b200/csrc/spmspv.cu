// spmspv.cu -- TileSpMSpV y = A x (Sec 3.3,
// P:790-863, Fig 4; semirings P:1373-1379).
//
// Three kernels on the caller's stream:
//   k_xscan    (a2) x -> tiled sparse vector: one thread per x entry finds the
//              non-empty nt-segments (x must be ascending so the
//              segments are runs), their nt-bit masks, the tile work
//              (tiles in tile column J) and the side work (side nonzeros of
//              column j); one decoupled look-back scan gives list positions,
//              work prefixes and the chunk -> entry maps of the expand kernel.
//   k_expand   (a3-a5) persistent, load balanced: warps pull 128-item chunks
//              of tile work and side work.  Tile item: intersect the tile's
//              column mask with the segment mask (skips the tile without
//              touching its nonzeros), multiply the hit columns'
//              nonzeros, accumulate into acc[m] with RED atomics and mark the
//              row in the touched bitmap.  Side item: one side nonzero.
//   k_compact  (a6) one thread per 32-row bitmap word: popc + look-back scan
//              -> y_idx ascending, y_val; acc and bits cleared as read.
#include "device.cuh"

namespace tsmv {

namespace {

template <int NT, class XV>
__global__ void __launch_bounds__(SCAN_BLOCK)
k_xscan(const int32_t *__restrict__ x_idx, const XV *__restrict__ x_val, long long k, long long n,
        const long long *__restrict__ tptr, const long long *__restrict__ sptr, ListsView Lv,
        Counters *__restrict__ cnt, LBDesc<4> *__restrict__ desc, unsigned epoch) {
    constexpr int LOG = Tr<NT>::LOG;
    using BS = cub::BlockScan<Quad, SCAN_BLOCK>;
    __shared__ typename BS::TempStorage ts;
    __shared__ unsigned s_bid;
    __shared__ long long s_pre[4];
    if (threadIdx.x == 0) s_bid = atomicAdd(&cnt->bid_scan, 1u);
    __syncthreads();
    const unsigned bid = s_bid;
    const long long e = (long long)bid * SCAN_BLOCK + threadIdx.x;
    Quad q = {{0, 0, 0, 0}};
    long long j = -1, seg = -1, wt = 0, ws = 0;
    bool head = false;
    double xvd = 1.0;
    if (e < k) {
        j = x_idx[e];
        long long prev = e > 0 ? (long long)x_idx[e - 1] : -1;
        bool bad = j < 0 || j >= n || prev >= j;
        if (bad) {
            cnt->err = 1;
        } else {
            seg = j >> LOG;
            head = e == 0 || (prev >> LOG) != seg;
            if (head) wt = tptr[seg + 1] - tptr[seg];
            ws = sptr[j + 1] - sptr[j];
        }
        if (x_val) xvd = (double)x_val[e];
        Lv.xv[e] = xvd;
    }
    q.v[0] = (head && wt > 0) ? 1 : 0;
    q.v[1] = head ? wt : 0;
    q.v[2] = ws > 0 ? 1 : 0;
    q.v[3] = ws;
    Quad ex, agg;
    BS(ts).ExclusiveScan(q, ex, Quad{{0, 0, 0, 0}}, QuadSum(), agg);
    if (threadIdx.x == 0) {
        long long pre[4];
        lookback<4>(desc, bid, epoch, agg.v, pre);
#pragma unroll
        for (int i = 0; i < 4; ++i) s_pre[i] = pre[i];
    }
    __syncthreads();
#pragma unroll
    for (int i = 0; i < 4; ++i) ex.v[i] += s_pre[i];
    if (head && wt > 0) {
        long long i = ex.v[0];
        unsigned long long mk = 0;
        for (long long e2 = e; e2 < k; ++e2) {
            long long j2 = x_idx[e2];
            if ((j2 >> LOG) != seg) break;
            mk |= 1ull << (j2 & (NT - 1));
        }
        Lv.Lt_seg[i] = seg;
        Lv.Lt_mask[i] = mk;
        Lv.Lt_first[i] = e;
        Lv.Lt_tbeg[i] = tptr[seg];
        Lv.Lt_wpre[i] = ex.v[1];
        write_chunks(Lv.Ct, ex.v[1], wt, (int)i);
    }
    if (ws > 0) {
        long long i = ex.v[2];
        Lv.Ls_beg[i] = sptr[j];
        Lv.Ls_wpre[i] = ex.v[3];
        Lv.Ls_x[i] = xvd;
        Lv.Ls_col[i] = (int)j;
        write_chunks(Lv.Cs, ex.v[3], ws, (int)i);
    }
    if (bid == gridDim.x - 1 && threadIdx.x == SCAN_BLOCK - 1) {
        long long tot[4];
#pragma unroll
        for (int i = 0; i < 4; ++i) tot[i] = s_pre[i] + agg.v[i];
        cnt->nLt = tot[0];
        cnt->Wt = tot[1];
        cnt->nLs = tot[2];
        cnt->Ws = tot[3];
        cnt->nCt = (tot[1] + CHUNK - 1) >> CHUNK_LOG;
        cnt->nCs = (tot[3] + CHUNK - 1) >> CHUNK_LOG;
        Lv.Lt_wpre[tot[0]] = tot[1];
        Lv.Ls_wpre[tot[2]] = tot[3];
        cnt->chunk_next = 0;
        cnt->bid_scan = 0;
    }
}

struct TileView {
    const long long *ptr;
    const int *trow;
    const void *mask;
    const long long *off;
    const void *idx;
    const void *val;
    const long long *sptr;
    const int *srow;
    const void *sval;
};

template <int SR>
__device__ __forceinline__ void accumulate(double *acc, uint32_t *rowbits, long long row, double a, double x) {
    if constexpr (SR == TSMV_PLUS_TIMES) {
        atomicAdd(&acc[row], a * x);
    } else if constexpr (SR == TSMV_MIN_SECOND) {
        atomicMax((unsigned long long *)&acc[row], ~ord_key(x));
    }
    atomicOr(&rowbits[row >> 5], 1u << (row & 31));
}

template <int NT, class AV, int SR>
__global__ void __launch_bounds__(256)
k_expand(TileView A, ListsView Lv, Counters *__restrict__ cnt, double *__restrict__ acc,
         uint32_t *__restrict__ rowbits) {
    using word_t = typename Tr<NT>::word_t;
    using idx_t = typename Tr<NT>::idx_t;
    constexpr int LOG = Tr<NT>::LOG;
    __shared__ long long win_all[8][CHUNK + 1];
    if (cnt->err) return;
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    long long *win = win_all[wid];
    const long long nCt = cnt->nCt, nCs = cnt->nCs;
    const long long nLt = cnt->nLt, nLs = cnt->nLs, Wt = cnt->Wt, Ws = cnt->Ws;
    const word_t *mask = (const word_t *)A.mask;
    const idx_t *idx = (const idx_t *)A.idx;
    const AV *val = (const AV *)A.val;
    const AV *sval = (const AV *)A.sval;
    while (true) {
        unsigned ch = 0;
        if (lane == 0) ch = atomicAdd(&cnt->chunk_next, 1u);
        ch = __shfl_sync(0xffffffffu, ch, 0);
        if (ch < nCt) {
            const long long s0 = Lv.Ct[ch];
            const long long base = (long long)ch << CHUNK_LOG;
            load_window(win, Lv.Lt_wpre, s0, nLt, lane);
#pragma unroll
            for (int u = 0; u < CHUNK / 32; ++u) {
                long long i = base + lane + 32 * u;
                if (i >= Wt) break;
                int q = window_find(win, i);
                long long s = s0 + q;
                long long t = Lv.Lt_tbeg[s] + (i - win[q]);
                unsigned long long xm = Lv.Lt_mask[s];
                word_t hit = mask[t] & (word_t)xm;
                if (hit) {
                    long long I = A.trow[t];
                    long long p0 = A.off[t], p1 = A.off[t + 1];
                    long long first = Lv.Lt_first[s];
                    for (long long p = p0; p < p1; ++p) {
                        unsigned id = idx[p];
                        unsigned cc = id >> LOG;
                        if ((hit >> cc) & 1) {
                            unsigned r = id & (NT - 1);
                            unsigned long long below = cc ? (xm & ((1ull << cc) - 1)) : 0ull;
                            double xv = Lv.xv[first + __popcll(below)];
                            double a = val ? (double)val[p] : 1.0;
                            accumulate<SR>(acc, rowbits, I * NT + r, a, xv);
                        }
                    }
                }
            }
            __syncwarp();
        } else if (ch < nCt + nCs) {
            const long long c2 = ch - nCt;
            const long long s0 = Lv.Cs[c2];
            const long long base = c2 << CHUNK_LOG;
            load_window(win, Lv.Ls_wpre, s0, nLs, lane);
#pragma unroll
            for (int u = 0; u < CHUNK / 32; ++u) {
                long long i = base + lane + 32 * u;
                if (i >= Ws) break;
                int q = window_find(win, i);
                long long s = s0 + q;
                long long p = Lv.Ls_beg[s] + (i - win[q]);
                long long row = A.srow[p];
                double a = sval ? (double)sval[p] : 1.0;
                accumulate<SR>(acc, rowbits, row, a, Lv.Ls_x[s]);
            }
            __syncwarp();
        } else {
            break;
        }
    }
}

template <class YV, int SR>
__global__ void __launch_bounds__(SCAN_BLOCK)
k_compact(uint32_t *__restrict__ rowbits, long long W, double *__restrict__ acc, long long row_begin,
          int32_t *__restrict__ y_idx, YV *__restrict__ y_val, long long y_cap, Counters *__restrict__ cnt,
          Counters *__restrict__ hmirror, LBDesc<1> *__restrict__ desc, unsigned epoch) {
    using BS = cub::BlockScan<long long, SCAN_BLOCK>;
    __shared__ typename BS::TempStorage ts;
    __shared__ unsigned s_bid;
    __shared__ long long s_pre;
    if (threadIdx.x == 0) s_bid = atomicAdd(&cnt->bid_compact, 1u);
    __syncthreads();
    const unsigned bid = s_bid;
    const long long w = (long long)bid * SCAN_BLOCK + threadIdx.x;
    unsigned bits = w < W ? rowbits[w] : 0u;
    long long c = __popc(bits), ex, agg;
    BS(ts).ExclusiveSum(c, ex, agg);
    if (threadIdx.x == 0) {
        long long pre;
        lookback<1>(desc, bid, epoch, &agg, &pre);
        s_pre = pre;
    }
    __syncthreads();
    long long pos = s_pre + ex;
    if (bits) {
        rowbits[w] = 0u;
        while (bits) {
            int b = __ffs(bits) - 1;
            bits &= bits - 1;
            long long row = w * 32 + b;
            double v = acc[row];
            acc[row] = 0.0;
            if (pos < y_cap) {
                y_idx[pos] = (int32_t)(row + row_begin);
                if (y_val) {
                    if constexpr (SR == TSMV_MIN_SECOND) v = ord_val(~(unsigned long long)__double_as_longlong(v));
                    y_val[pos] = (YV)v;
                }
            }
            ++pos;
        }
    }
    if (bid == gridDim.x - 1 && threadIdx.x == SCAN_BLOCK - 1) {
        long long tot = s_pre + agg;
        cnt->y_nnz = tot;
        hmirror->y_nnz = tot;
        hmirror->err = cnt->err;
        hmirror->nLt = cnt->nLt;
        hmirror->Wt = cnt->Wt;
        hmirror->nLs = cnt->nLs;
        hmirror->Ws = cnt->Ws;
        cnt->err = 0;
        cnt->bid_compact = 0;
    }
}

inline TileView tile_view(const TileSet &S) {
    TileView v;
    v.ptr = S.ptr.as<long long>();
    v.trow = S.trow.as<int>();
    v.mask = S.mask.p;
    v.off = S.off.as<long long>();
    v.idx = S.idx.p;
    v.val = S.has_vals ? S.val.p : nullptr;
    v.sptr = S.sptr.as<long long>();
    v.srow = S.srow.as<int>();
    v.sval = S.has_vals ? S.sval.p : nullptr;
    return v;
}

template <int NT, class AV, int SR>
void launch_expand(tsmv_ctx *c, cudaStream_t st) {
    k_expand<NT, AV, SR><<<c->expand_blocks, 256, 0, st>>>(tile_view(c->P), lists_view(c),
                                                           c->counters.as<Counters>(), c->acc.as<double>(),
                                                           c->rowbits.as<uint32_t>());
}

template <int NT, class AV>
void launch_expand_sr(tsmv_ctx *c, int sr, cudaStream_t st) {
    if (sr == TSMV_PLUS_TIMES) launch_expand<NT, AV, TSMV_PLUS_TIMES>(c, st);
    else if (sr == TSMV_OR_AND) launch_expand<NT, AV, TSMV_OR_AND>(c, st);
    else launch_expand<NT, AV, TSMV_MIN_SECOND>(c, st);
}

template <int NT>
void launch_xscan(tsmv_ctx *c, const int32_t *xi, const void *xv, bool f32, long long k, cudaStream_t st) {
    int grid = (int)((k + SCAN_BLOCK - 1) / SCAN_BLOCK);
    if (f32)
        k_xscan<NT, float><<<grid, SCAN_BLOCK, 0, st>>>(xi, (const float *)xv, k, c->n, c->P.ptr.as<long long>(),
                                                        c->P.sptr.as<long long>(), lists_view(c),
                                                        c->counters.as<Counters>(),
                                                        c->L.desc_scan.as<LBDesc<4>>(), c->epoch);
    else
        k_xscan<NT, double><<<grid, SCAN_BLOCK, 0, st>>>(xi, (const double *)xv, k, c->n,
                                                         c->P.ptr.as<long long>(), c->P.sptr.as<long long>(),
                                                         lists_view(c), c->counters.as<Counters>(),
                                                         c->L.desc_scan.as<LBDesc<4>>(), c->epoch);
}

template <class YV>
void launch_compact(tsmv_ctx *c, int sr, int32_t *yi, void *yv, long long ycap, cudaStream_t st) {
    long long W = (c->m + 31) / 32;
    int grid = (int)std::max<long long>(1, (W + SCAN_BLOCK - 1) / SCAN_BLOCK);
    auto *d = c->desc_compact.as<LBDesc<1>>();
    if (sr == TSMV_MIN_SECOND)
        k_compact<YV, TSMV_MIN_SECOND><<<grid, SCAN_BLOCK, 0, st>>>(
            c->rowbits.as<uint32_t>(), W, c->acc.as<double>(), c->row_begin, yi, (YV *)yv, ycap,
            c->counters.as<Counters>(), c->hcnt_dev, d, c->epoch);
    else
        k_compact<YV, TSMV_PLUS_TIMES><<<grid, SCAN_BLOCK, 0, st>>>(
            c->rowbits.as<uint32_t>(), W, c->acc.as<double>(), c->row_begin, yi,
            sr == TSMV_OR_AND ? nullptr : (YV *)yv, ycap, c->counters.as<Counters>(), c->hcnt_dev, d, c->epoch);
}

}  // namespace

int expand_occupancy(int nt, int dtype) {
    int b = 0;
    bool f32 = dtype == TSMV_F32;
    cudaError_t e;
    if (nt == 16) e = f32 ? cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, k_expand<16, float, 0>, 256, 0)
                          : cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, k_expand<16, double, 0>, 256, 0);
    else if (nt == 32) e = f32 ? cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, k_expand<32, float, 0>, 256, 0)
                               : cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, k_expand<32, double, 0>, 256, 0);
    else e = f32 ? cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, k_expand<64, float, 0>, 256, 0)
                 : cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, k_expand<64, double, 0>, 256, 0);
    if (e != cudaSuccess || b < 1) {
        cudaGetLastError();
        b = 4;
    }
    return b;
}

void ensure_lists(tsmv_ctx *c, int64_t k) {
    Lists &L = c->L;
    if (k > L.cap_ent) {
        int64_t cap = std::max<int64_t>(k, 1024);
        int64_t segs = std::min<int64_t>(cap, c->nTC);
        L.Lt_seg.alloc((segs + 1) * 8);
        L.Lt_mask.alloc((segs + 1) * 8);
        L.Lt_first.alloc((segs + 1) * 8);
        L.Lt_tbeg.alloc((segs + 1) * 8);
        L.Lt_wpre.alloc((segs + 1) * 8);
        L.Ls_beg.alloc((cap + 1) * 8);
        L.Ls_wpre.alloc((cap + 1) * 8);
        L.Ls_x.alloc((cap + 1) * 8);
        L.Ls_col.alloc((cap + 1) * 4);
        L.xv.alloc((cap + 1) * 8);
        int64_t blocks = (cap + SCAN_BLOCK - 1) / SCAN_BLOCK + 1;
        L.desc_scan.alloc(blocks * sizeof(LBDesc<4>));
        TSMV_CUDA(cudaMemset(L.desc_scan.p, 0, blocks * sizeof(LBDesc<4>)));
        L.cap_ent = cap;
        L.cap_seg = segs;
    }
    if (L.cap_ct == 0) {
        // work items are bounded by the tile / side totals
        int64_t nct = (c->P.T + CHUNK - 1) / CHUNK + 2;
        int64_t ncs = (c->P.side_nnz + CHUNK - 1) / CHUNK + 2;
        L.Ct.alloc(nct * 4);
        L.Cs.alloc(ncs * 4);
        L.cap_ct = nct;
        L.cap_cs = ncs;
    }
}

// Debug aid (TSMV_CHECK_LISTS=1): validate the k_xscan lists on the host.
void debug_check_lists(tsmv_ctx *c, cudaStream_t st) {
    TSMV_CUDA(cudaStreamSynchronize(st));
    Counters h;
    TSMV_CUDA(cudaMemcpy(&h, c->counters.p, sizeof(h), cudaMemcpyDeviceToHost));
    auto chk = [&](const char *nm, const DevBuf &wpre_b, const DevBuf &C_b, long long nL, long long W, long long nC) {
        std::vector<long long> wpre(nL + 1);
        std::vector<int> C(nC);
        TSMV_CUDA(cudaMemcpy(wpre.data(), wpre_b.p, (nL + 1) * 8, cudaMemcpyDeviceToHost));
        if (nC) TSMV_CUDA(cudaMemcpy(C.data(), C_b.p, nC * 4, cudaMemcpyDeviceToHost));
        int bad = 0;
        if (nL && wpre[0] != 0) fprintf(stderr, "[%s] wpre[0]=%lld\n", nm, wpre[0]), ++bad;
        if (wpre[nL] != W) fprintf(stderr, "[%s] sentinel %lld != W %lld\n", nm, wpre[nL], W), ++bad;
        for (long long i = 0; i + 1 <= nL && bad < 10; ++i)
            if (wpre[i + 1] <= wpre[i]) fprintf(stderr, "[%s] wpre[%lld]=%lld wpre[+1]=%lld\n", nm, i, wpre[i], wpre[i + 1]), ++bad;
        for (long long ch = 0; ch < nC && bad < 20; ++ch) {
            long long it = ch << CHUNK_LOG, s = C[ch];
            if (s < 0 || s >= nL || !(wpre[s] <= it && it < wpre[s + 1]))
                fprintf(stderr, "[%s] chunk %lld -> %lld wrong\n", nm, ch, s), ++bad;
        }
        fprintf(stderr, "[%s] nL=%lld W=%lld nC=%lld bad=%d\n", nm, nL, W, nC, bad);
    };
    chk("tile", c->L.Lt_wpre, c->L.Ct, h.nLt, h.Wt, h.nCt);
    chk("side", c->L.Ls_wpre, c->L.Cs, h.nLs, h.Ws, h.nCs);
}

}  // namespace tsmv

using namespace tsmv;

extern "C" tsmv_status tsmv_spmspv(tsmv_ctx *c, tsmv_semiring sr, int64_t x_nnz, const int32_t *x_idx,
                                   const void *x_val, int64_t y_cap, int32_t *y_idx, void *y_val, int64_t *y_nnz,
                                   void *cuda_stream) {
    try {
        TSMV_REQUIRE(c != nullptr, "tsmv_spmspv: NULL ctx");
        TSMV_REQUIRE(y_nnz != nullptr, "tsmv_spmspv: NULL y_nnz");
        TSMV_REQUIRE(sr >= 0 && sr <= 2, "tsmv_spmspv: bad semiring %d", (int)sr);
        TSMV_REQUIRE(x_nnz >= 0 && x_nnz <= c->n, "tsmv_spmspv: x_nnz %lld out of [0, ncols]", (long long)x_nnz);
        TSMV_REQUIRE(x_nnz == 0 || x_idx != nullptr, "tsmv_spmspv: NULL x_idx");
        TSMV_REQUIRE(sr == TSMV_OR_AND || x_nnz == 0 || x_val != nullptr, "tsmv_spmspv: NULL x_val");
        TSMV_REQUIRE(y_cap >= 0, "tsmv_spmspv: negative y_cap");
        TSMV_REQUIRE(y_cap == 0 || y_idx != nullptr, "tsmv_spmspv: NULL y_idx");
        TSMV_REQUIRE(sr == TSMV_OR_AND || y_cap == 0 || y_val != nullptr, "tsmv_spmspv: NULL y_val");
        TSMV_CUDA(cudaSetDevice(c->device));
        cudaStream_t st = (cudaStream_t)cuda_stream;
        *y_nnz = 0;
        if (x_nnz == 0) {
            c->hcnt->nLt = c->hcnt->Wt = c->hcnt->nLs = c->hcnt->Ws = c->hcnt->y_nnz = 0;
            return TSMV_OK;
        }
        const bool f32 = c->dtype == TSMV_F32;
        const size_t vb = f32 ? 4 : 8;
        // stage host inputs
        const int32_t *xi = x_idx;
        const void *xv = (sr == TSMV_OR_AND) ? nullptr : x_val;
        if (!is_device_ptr(xi)) {
            c->stage_x_idx.ensure(x_nnz * 4);
            TSMV_CUDA(cudaMemcpyAsync(c->stage_x_idx.p, xi, x_nnz * 4, cudaMemcpyHostToDevice, st));
            xi = c->stage_x_idx.as<int32_t>();
        }
        if (xv && !is_device_ptr(xv)) {
            c->stage_x_val.ensure(x_nnz * vb);
            TSMV_CUDA(cudaMemcpyAsync(c->stage_x_val.p, xv, x_nnz * vb, cudaMemcpyHostToDevice, st));
            xv = c->stage_x_val.p;
        }
        bool host_y = (y_cap > 0) && !is_device_ptr(y_idx);
        bool host_yv = (y_cap > 0) && sr != TSMV_OR_AND && y_val && !is_device_ptr(y_val);
        int32_t *yi = y_idx;
        void *yv = (sr == TSMV_OR_AND) ? nullptr : y_val;
        int64_t ycap_dev = y_cap;
        if (host_y || host_yv) ycap_dev = std::min<int64_t>(y_cap, c->m);
        if (host_y) {
            c->stage_y_idx.ensure(std::max<int64_t>(ycap_dev, 1) * 4);
            yi = c->stage_y_idx.as<int32_t>();
        }
        if (host_yv) {
            c->stage_y_val.ensure(std::max<int64_t>(ycap_dev, 1) * vb);
            yv = c->stage_y_val.p;
        }
        ensure_lists(c, x_nnz);
        c->epoch++;
        switch (c->nt) {
            case 16: launch_xscan<16>(c, xi, xv, f32, x_nnz, st); break;
            case 32: launch_xscan<32>(c, xi, xv, f32, x_nnz, st); break;
            default: launch_xscan<64>(c, xi, xv, f32, x_nnz, st); break;
        }
        TSMV_CUDA(cudaGetLastError());
        if (getenv("TSMV_CHECK_LISTS")) debug_check_lists(c, st);
        if (f32) {
            switch (c->nt) {
                case 16: launch_expand_sr<16, float>(c, sr, st); break;
                case 32: launch_expand_sr<32, float>(c, sr, st); break;
                default: launch_expand_sr<64, float>(c, sr, st); break;
            }
        } else {
            switch (c->nt) {
                case 16: launch_expand_sr<16, double>(c, sr, st); break;
                case 32: launch_expand_sr<32, double>(c, sr, st); break;
                default: launch_expand_sr<64, double>(c, sr, st); break;
            }
        }
        TSMV_CUDA(cudaGetLastError());
        if (f32) launch_compact<float>(c, sr, yi, yv, ycap_dev, st);
        else launch_compact<double>(c, sr, yi, yv, ycap_dev, st);
        TSMV_CUDA(cudaGetLastError());
        TSMV_CUDA(cudaStreamSynchronize(st));
        volatile Counters *h = c->hcnt;
        int64_t ynnz = h->y_nnz;
        int err = h->err;
        TSMV_REQUIRE(err == 0, "tsmv_spmspv: x indices must be strictly ascending and in [0, %lld)",
                     (long long)c->n);
        *y_nnz = ynnz;
        if (ynnz > y_cap) {
            set_error("tsmv_spmspv: y_cap %lld < y_nnz %lld", (long long)y_cap, (long long)ynnz);
            return TSMV_ECAPACITY;
        }
        if (host_y) TSMV_CUDA(cudaMemcpyAsync(y_idx, yi, ynnz * 4, cudaMemcpyDeviceToHost, st));
        if (host_yv) TSMV_CUDA(cudaMemcpyAsync(y_val, yv, ynnz * vb, cudaMemcpyDeviceToHost, st));
        if (host_y || host_yv) TSMV_CUDA(cudaStreamSynchronize(st));
        return TSMV_OK;
    } catch (const Err &e) {
        return e.st;
    }
}

extern "C" tsmv_status tsmv_last_call_stats(tsmv_ctx *c, tsmv_call_stats *s) {
    try {
        TSMV_REQUIRE(c && s, "tsmv_last_call_stats: NULL argument");
        volatile Counters *h = c->hcnt;
        s->x_nnz = 0;
        s->x_segments = h->nLt;
        s->tile_items = h->Wt;
        s->side_items = h->Ws;
        s->y_nnz = h->y_nnz;
        return TSMV_OK;
    } catch (const Err &e) {
        return e.st;
    }
}
