// spmspv.cu -- TileSpMSpV y = A x (Sec 3.3,
// P:790-863, Fig 4; semirings P:1373-1379).
//
// ONE cooperative persistent kernel per call (one CTA of 1024 threads per SM),
// phases separated by grid barriers instead of kernel boundaries:
//   A  (a2) x -> tiled sparse vector.  x is strictly ascending, so the
//           non-empty nt-segments are runs of x; each CTA takes a
//           slice of x, finds segment heads, their nt-bit masks, the tile work
//           (tiles in tile column J) and the side work (side nonzeros of each
//           column j), writes x_j into xd[j] (the paper's x_tile, addressed by
//           column instead of through x_ptr), and publishes its totals.
//   -- barrier --  every CTA scans the <= #SM totals itself (no look-back chain)
//   A' writes the segment list / side list, their work prefixes and the
//           chunk -> entry maps of the load balancer.
//   -- barrier --
//   B  (a3-a5) warps take 128-item chunks (first chunk static, then an atomic
//           queue).  Tile item: AND the tile's column mask with the segment
//           mask (a miss never touches the tile); a hit loads one
//           16-byte descriptor + the column start offsets and multiplies only
//           the hit columns' nonzeros.  Side item: one side nonzero (CSC column
//           merge, Alg 2).  Accumulation: RED.ADD.F64 into acc[m] + touched bit.
//   -- barrier --
//   C  (a6) CTAs count the set bits of their slice of the touched bitmap,
//   -- barrier --  then write y (ascending) with a "transposed" warp walk: lane l
//           handles bit l of each word, so a dense stretch of y costs one round
//           of 32 parallel accumulator loads per word.  acc/bits cleared on read.
#include "device.cuh"

namespace tsmv {

namespace {

constexpr int FB = 512;  // threads per CTA of the fused kernel
constexpr int TRING = 4096;

struct FusedArgs {
    const int32_t *x_idx;
    const void *x_val;
    long long k, n, m, W, row_begin;
    // tiles (push format)
    const long long *tptr;
    const void *mask;
    const void *idx;
    const void *val;
    const void *desc;
    const void *cstart;
    const long long *sptr;
    const int *srow;
    const void *sval;
    ListsView Lv;
    double *acc;
    uint32_t *rowbits;
    long long *partials;  // [G][8]
    long long *acct;      // [G][4]
    int32_t *y_idx;
    void *y_val;
    long long y_cap;
    long long *ynnz_dev;
    Counters *cnt;
    Counters *hm;
    unsigned long long bar_base;
    unsigned long long *tring;  // nullptr = no timing
    long long tslot;
};

template <int SR>
__device__ __forceinline__ void accumulate(double *acc, uint32_t *rowbits, long long row, double a, double x) {
    if constexpr (SR == TSMV_PLUS_TIMES) {
        atomicAdd(&acc[row], a * x);
    } else if constexpr (SR == TSMV_MIN_SECOND) {
        atomicMax((unsigned long long *)&acc[row], ~ord_key(x));
    }
    // Touched-row bit: test before set.  Power-law rows receive thousands of
    // contributions per call; an unconditional RED.OR on their (shared) word
    // serialises in one L2 slice.  A stale read only costs a redundant RED.
    const unsigned bit = 1u << (row & 31);
    unsigned *wp = &rowbits[row >> 5];
    if (!(__ldca(wp) & bit)) atomicOr(wp, bit);
}

// per-entry facts of phase A
template <int NT>
__device__ __forceinline__ void entry_facts(const int32_t *x_idx, long long e, long long k, long long n,
                                            const long long *tptr, const long long *sptr, long long &j,
                                            long long &seg, bool &head, long long &wt, long long &ws, bool &bad) {
    constexpr int LOG = Tr<NT>::LOG;
    j = x_idx[e];
    const long long prev = e > 0 ? (long long)x_idx[e - 1] : -1;
    bad = j < 0 || j >= n || prev >= j;
    head = false;
    wt = ws = 0;
    seg = j >> LOG;
    if (!bad) {
        head = e == 0 || (prev >> LOG) != seg;
        if (head) wt = tptr[seg + 1] - tptr[seg];
        ws = sptr[j + 1] - sptr[j];
    }
}

template <int NT, class AV, class XV, int SR>
__global__ void __launch_bounds__(FB, 1) k_spmspv_fused(FusedArgs a) {
    using word_t = typename Tr<NT>::word_t;
    using idx_t = typename Tr<NT>::idx_t;
    using cs_t = typename Tr<NT>::cs_t;
    constexpr int LOG = Tr<NT>::LOG;
    constexpr int U = CHUNK / 32;
    constexpr int NW = FB / 32;
    using BSQ = cub::BlockScan<Quad, FB>;
    using BSL = cub::BlockScan<long long, FB>;
    __shared__ union {
        typename BSQ::TempStorage q;
        typename BSL::TempStorage l;
    } ts;
    __shared__ long long win_all[NW][CHUNK + 1];
    __shared__ long long s_pre[4], s_tot[4];
    __shared__ long long s_acct[NW][3];
    __shared__ int s_err;
    const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
    const int G = gridDim.x, b = blockIdx.x;
    unsigned long long target = a.bar_base;
    const bool stamp = a.tring && b == 0 && tid == 0;
    unsigned long long *ts_out = a.tring ? a.tring + (a.tslot % TRING) * 8 : nullptr;
    if (stamp) ts_out[0] = globaltimer_ns();

    // ------------------------------------------------------------ phase A: x -> segments
    const long long E = (a.k + G - 1) / G;
    const long long e0 = (long long)b * E, e1 = min(a.k, e0 + E);
    const long long per = (E + FB - 1) / FB;
    const long long te0 = min(e1, e0 + tid * per), te1 = min(e1, te0 + per);
    Quad q = {{0, 0, 0, 0}};
    bool any_bad = false;
    for (long long e = te0; e < te1; ++e) {
        long long j, seg, wt, ws;
        bool head, bad;
        entry_facts<NT>(a.x_idx, e, a.k, a.n, a.tptr, a.sptr, j, seg, head, wt, ws, bad);
        any_bad |= bad;
        q.v[0] += (head && wt > 0);
        q.v[1] += wt;
        q.v[2] += (ws > 0);
        q.v[3] += ws;
        if (!bad) {
            double xv = a.x_val ? (double)((const XV *)a.x_val)[e] : 1.0;
            a.Lv.xd[j] = xv;
        }
    }
    if (any_bad) a.cnt->err = 1;
    Quad ex, agg;
    BSQ(ts.q).ExclusiveScan(q, ex, Quad{{0, 0, 0, 0}}, QuadSum(), agg);
    if (tid < 4) a.partials[b * 8 + tid] = agg.v[tid];
    if (b == 0 && tid == 0) a.cnt->chunk_next = 0;
    grid_sync(&a.cnt->bar, target);
    if (stamp) ts_out[1] = globaltimer_ns();

    // every CTA reduces the G partials itself: prefix of CTAs < b, and totals
    if (tid < 32) {
        long long pre[4] = {0, 0, 0, 0}, tot[4] = {0, 0, 0, 0};
        for (int g = lane; g < G; g += 32) {
#pragma unroll
            for (int i = 0; i < 4; ++i) {
                long long v = __ldcg(&a.partials[g * 8 + i]);
                tot[i] += v;
                if (g < b) pre[i] += v;
            }
        }
#pragma unroll
        for (int i = 0; i < 4; ++i) {
#pragma unroll
            for (int o = 16; o > 0; o >>= 1) {
                pre[i] += __shfl_xor_sync(0xffffffffu, pre[i], o);
                tot[i] += __shfl_xor_sync(0xffffffffu, tot[i], o);
            }
        }
        if (lane == 0) {
#pragma unroll
            for (int i = 0; i < 4; ++i) {
                s_pre[i] = pre[i];
                s_tot[i] = tot[i];
            }
            s_err = __ldcg(&a.cnt->err);
        }
    }
    __syncthreads();
    const bool err = s_err != 0;
    // A': write the lists
    if (!err) {
        long long oLt = s_pre[0] + ex.v[0], oWt = s_pre[1] + ex.v[1];
        long long oLs = s_pre[2] + ex.v[2], oWs = s_pre[3] + ex.v[3];
        for (long long e = te0; e < te1; ++e) {
            long long j, seg, wt, ws;
            bool head, bad;
            entry_facts<NT>(a.x_idx, e, a.k, a.n, a.tptr, a.sptr, j, seg, head, wt, ws, bad);
            if (head && wt > 0) {
                unsigned long long mk = 0;
                for (long long e2 = e; e2 < a.k; ++e2) {
                    const long long j2 = a.x_idx[e2];
                    if ((j2 >> LOG) != seg) break;
                    mk |= 1ull << (j2 & (NT - 1));
                }
                a.Lv.Lt_seg[oLt] = seg;
                a.Lv.Lt_mask[oLt] = mk;
                a.Lv.Lt_tbeg[oLt] = a.tptr[seg];
                a.Lv.Lt_wpre[oLt] = oWt;
                write_chunks(a.Lv.Ct, oWt, wt, (int)oLt);
                ++oLt;
                oWt += wt;
            }
            if (ws > 0) {
                a.Lv.Ls_beg[oLs] = a.sptr[j];
                a.Lv.Ls_wpre[oLs] = oWs;
                a.Lv.Ls_x[oLs] = a.x_val ? (double)((const XV *)a.x_val)[e] : 1.0;
                write_chunks(a.Lv.Cs, oWs, ws, (int)oLs);
                ++oLs;
                oWs += ws;
            }
        }
        if (b == G - 1 && tid == 0) {
            a.Lv.Lt_wpre[s_tot[0]] = s_tot[1];
            a.Lv.Ls_wpre[s_tot[2]] = s_tot[3];
        }
    }
    grid_sync(&a.cnt->bar, target);
    if (stamp) ts_out[2] = globaltimer_ns();

    // ------------------------------------------------------------ phase B: expand
    long long n_hit = 0, n_hcol = 0, n_mac = 0;
    if (!err) {
        const long long nLt = s_tot[0], Wt = s_tot[1], nLs = s_tot[2], Ws = s_tot[3];
        const long long nCt = (Wt + CHUNK - 1) >> CHUNK_LOG, nCs = (Ws + CHUNK - 1) >> CHUNK_LOG;
        long long *win = win_all[wid];
        const word_t *mask = (const word_t *)a.mask;
        const idx_t *idx = (const idx_t *)a.idx;
        const AV *val = (const AV *)a.val;
        const AV *sval = (const AV *)a.sval;
        const cs_t *cstart = (const cs_t *)a.cstart;
        const unsigned nwarps = (unsigned)(G * NW);
        unsigned ch = (unsigned)(b * NW + wid);  // first chunk static, then the queue
        while (true) {
            if (ch < nCt) {
                const long long s0 = __ldcg(&a.Lv.Ct[ch]);
                const long long base = (long long)ch << CHUNK_LOG;
                load_window(win, a.Lv.Lt_wpre, s0, nLt, lane);
                long long sidx[U], t[U];
                bool ok[U];
#pragma unroll
                for (int u = 0; u < U; ++u) {
                    const long long i = base + lane + 32 * u;
                    ok[u] = i < Wt;
                    const int qq = ok[u] ? window_find(win, i) : 0;
                    sidx[u] = s0 + qq;
                    t[u] = i - win[qq];
                }
                long long J[U];
                word_t xm[U];
#pragma unroll
                for (int u = 0; u < U; ++u) {
                    if (ok[u]) {
                        t[u] += __ldcg(&a.Lv.Lt_tbeg[sidx[u]]);
                        xm[u] = (word_t)__ldcg(&a.Lv.Lt_mask[sidx[u]]);
                        J[u] = __ldcg(&a.Lv.Lt_seg[sidx[u]]);
                    }
                }
                word_t hit[U];
#pragma unroll
                for (int u = 0; u < U; ++u) hit[u] = ok[u] ? (word_t)(mask[t[u]] & xm[u]) : (word_t)0;
#pragma unroll
                for (int u = 0; u < U; ++u) {
                    if (hit[u]) {
                        const TileDesc d = ((const TileDesc *)a.desc)[t[u]];
                        ++n_hit;
                        word_t h = hit[u];
                        const long long rowbase = (long long)d.trow * NT;
                        while (h) {
                            const int c = ffs_w(h);
                            h &= h - 1;
                            const int p0 = cstart[t[u] * NT + c];
                            const int p1 = c + 1 < NT ? (int)cstart[t[u] * NT + c + 1] : d.nnz;
                            const double xv = __ldcg(&a.Lv.xd[J[u] * NT + c]);
                            for (int p = p0; p < p1; ++p) {
                                const unsigned r = idx[d.off + p] & (NT - 1);
                                const double av = val ? (double)val[d.off + p] : 1.0;
                                accumulate<SR>(a.acc, a.rowbits, rowbase + r, av, xv);
                            }
                            n_mac += p1 - p0;
                            ++n_hcol;
                        }
                    }
                }
            } else if (ch < nCt + nCs) {
                const long long c2 = (long long)ch - nCt;
                const long long s0 = __ldcg(&a.Lv.Cs[c2]);
                const long long base = c2 << CHUNK_LOG;
                load_window(win, a.Lv.Ls_wpre, s0, nLs, lane);
                long long p[U], sidx[U];
                bool ok[U];
#pragma unroll
                for (int u = 0; u < U; ++u) {
                    const long long i = base + lane + 32 * u;
                    ok[u] = i < Ws;
                    const int qq = ok[u] ? window_find(win, i) : 0;
                    sidx[u] = s0 + qq;
                    p[u] = i - win[qq];
                }
                double xv[U];
#pragma unroll
                for (int u = 0; u < U; ++u) {
                    if (ok[u]) {
                        p[u] += __ldcg(&a.Lv.Ls_beg[sidx[u]]);
                        xv[u] = __ldcg(&a.Lv.Ls_x[sidx[u]]);
                    }
                }
                long long row[U];
                double av[U];
#pragma unroll
                for (int u = 0; u < U; ++u) {
                    if (ok[u]) {
                        row[u] = a.srow[p[u]];
                        av[u] = sval ? (double)sval[p[u]] : 1.0;
                    }
                }
#pragma unroll
                for (int u = 0; u < U; ++u)
                    if (ok[u]) accumulate<SR>(a.acc, a.rowbits, row[u], av[u], xv[u]);
            } else {
                break;
            }
            __syncwarp();
            unsigned nx = 0;
            if (lane == 0) nx = nwarps + atomicAdd(&a.cnt->chunk_next, 1u);
            ch = __shfl_sync(0xffffffffu, nx, 0);
        }
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        n_hit += __shfl_xor_sync(0xffffffffu, n_hit, o);
        n_hcol += __shfl_xor_sync(0xffffffffu, n_hcol, o);
        n_mac += __shfl_xor_sync(0xffffffffu, n_mac, o);
    }
    if (lane == 0) {
        s_acct[wid][0] = n_hit;
        s_acct[wid][1] = n_hcol;
        s_acct[wid][2] = n_mac;
    }
    grid_sync(&a.cnt->bar, target);  // (its __syncthreads also orders s_acct)
    if (stamp) ts_out[3] = globaltimer_ns();
    if (tid < 3) {
        long long sum = 0;
        for (int w = 0; w < NW; ++w) sum += s_acct[w][tid];
        a.acct[b * 4 + tid] = sum;
    }

    // ------------------------------------------------------------ phase C: compact
    const long long S = (((a.W + G - 1) / G) + 31) & ~31ll;  // words per CTA, warp aligned
    const long long w0 = (long long)b * S, w1 = min(a.W, w0 + S);
    long long mycnt = 0;
    for (long long w = w0 + tid; w < w1; w += FB) mycnt += __popc(__ldcg(&a.rowbits[w]));
    long long blk = 0;
    {
        long long dummy;
        BSL(ts.l).ExclusiveSum(mycnt, dummy, blk);
    }
    if (tid == 0) a.partials[b * 8 + 4] = blk;
    grid_sync(&a.cnt->bar, target);
    if (stamp) ts_out[4] = globaltimer_ns();
    if (tid < 32) {
        long long pre = 0, tot = 0;
        for (int g = lane; g < G; g += 32) {
            long long v = __ldcg(&a.partials[g * 8 + 4]);
            tot += v;
            if (g < b) pre += v;
        }
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) {
            pre += __shfl_xor_sync(0xffffffffu, pre, o);
            tot += __shfl_xor_sync(0xffffffffu, tot, o);
        }
        if (lane == 0) {
            s_pre[0] = pre;
            s_tot[0] = tot;
        }
    }
    __syncthreads();
    long long carry = s_pre[0];
    const long long ycap = a.y_cap;
    const unsigned lt = (1u << lane) - 1;
    for (long long rb = w0; rb < w1; rb += FB) {
        const long long w = rb + tid;
        const unsigned bits = w < w1 ? __ldcg(&a.rowbits[w]) : 0u;
        long long c = __popc(bits), exw, rtot;
        BSL(ts.l).ExclusiveSum(c, exw, rtot);
        const long long pos0 = carry + exw;
        carry += rtot;
        if (bits) a.rowbits[w] = 0u;
        const long long wbase = w - lane;
        unsigned todo = __ballot_sync(0xffffffffu, bits != 0);
        while (todo) {
            int src[8];
            int nb = 0;
#pragma unroll
            for (int kk = 0; kk < 8; ++kk) {
                src[kk] = 0;
                if (todo) {
                    src[kk] = __ffs(todo) - 1;
                    todo &= todo - 1;
                    nb = kk + 1;
                }
            }
            unsigned wb[8];
            long long wp[8];
            double v[8];
            bool mine[8];
#pragma unroll
            for (int kk = 0; kk < 8; ++kk) {
                wb[kk] = __shfl_sync(0xffffffffu, bits, src[kk]);
                wp[kk] = __shfl_sync(0xffffffffu, pos0, src[kk]);
                mine[kk] = kk < nb && ((wb[kk] >> lane) & 1u);
                if (mine[kk]) v[kk] = __ldcg(&a.acc[(wbase + src[kk]) * 32 + lane]);
            }
#pragma unroll
            for (int kk = 0; kk < 8; ++kk) {
                if (mine[kk]) {
                    const long long row = (wbase + src[kk]) * 32 + lane;
                    const long long pos = wp[kk] + __popc(wb[kk] & lt);
                    a.acc[row] = 0.0;
                    if (pos < ycap) {
                        a.y_idx[pos] = (int32_t)(row + a.row_begin);
                        if (a.y_val) {
                            double x = v[kk];
                            if constexpr (SR == TSMV_MIN_SECOND)
                                x = ord_val(~(unsigned long long)__double_as_longlong(x));
                            ((XV *)a.y_val)[pos] = (XV)x;
                        }
                    }
                }
            }
        }
        __syncthreads();  // ts.l reuse
    }
    if (b == 0 && tid == 0) {
        // every CTA read cnt->err before barrier 3, so it can be reset here
        const long long tot = s_tot[0];
        a.cnt->y_nnz = tot;
        a.hm->y_nnz = tot;
        a.hm->err = err ? 1 : 0;
        if (a.ynnz_dev) *a.ynnz_dev = err ? -1 : tot;
        a.cnt->err = 0;
        if (a.tring) ts_out[5] = globaltimer_ns();
    }
}

// Phase-A totals / accounting for tsmv_last_call_stats are summed on the host
// from `partials` and `acct`.

template <int NT, class AV, class XV, int SR> void *fused_fn() {
    return (void *)k_spmspv_fused<NT, AV, XV, SR>;
}

template <int NT, class AV, class XV> void *pick_sr(int sr) {
    if (sr == TSMV_PLUS_TIMES) return fused_fn<NT, AV, XV, TSMV_PLUS_TIMES>();
    if (sr == TSMV_OR_AND) return fused_fn<NT, AV, XV, TSMV_OR_AND>();
    return fused_fn<NT, AV, XV, TSMV_MIN_SECOND>();
}

void *pick_kernel(int nt, bool f32, int sr) {
    // AV = matrix value type, XV = x / y value type (both fp32 for F32 contexts)
    if (f32) {
        if (nt == 16) return pick_sr<16, float, float>(sr);
        if (nt == 32) return pick_sr<32, float, float>(sr);
        return pick_sr<64, float, float>(sr);
    }
    if (nt == 16) return pick_sr<16, double, double>(sr);
    if (nt == 32) return pick_sr<32, double, double>(sr);
    return pick_sr<64, double, double>(sr);
}

}  // namespace

int expand_occupancy(int nt, int dtype) {
    // blocks per SM of the persistent BFS push kernels (256 threads)
    (void)nt;
    (void)dtype;
    return 4;
}

int fused_occupancy(int nt, int dtype) {
    int bps = 0;
    void *f = pick_kernel(nt, dtype == TSMV_F32, TSMV_PLUS_TIMES);
    cudaError_t e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&bps, f, FB, 0);
    if (e != cudaSuccess || bps < 1) {
        cudaGetLastError();
        bps = 0;
    }
    return bps;
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

// Enqueue one fused SpMSpV (device pointers only, no sync).
void enqueue_spmspv(tsmv_ctx *c, int sr, long long k, const int32_t *xi, const void *xv, long long ycap,
                    int32_t *yi, void *yv, long long *ynnz_dev, cudaStream_t st) {
    const bool f32 = c->dtype == TSMV_F32;
    ensure_lists(c, k);
    FusedArgs a;
    a.x_idx = xi;
    a.x_val = xv;
    a.k = k;
    a.n = c->n;
    a.m = c->m;
    a.W = (c->m + 31) / 32;
    a.row_begin = c->row_begin;
    a.tptr = c->P.ptr.as<long long>();
    a.mask = c->P.mask.p;
    a.idx = c->P.idx.p;
    a.val = c->P.has_vals ? c->P.val.p : nullptr;
    a.desc = c->P.desc.p;
    a.cstart = c->P.cstart.p;
    a.sptr = c->P.sptr.as<long long>();
    a.srow = c->P.srow.as<int>();
    a.sval = c->P.has_vals ? c->P.sval.p : nullptr;
    a.Lv = lists_view(c);
    a.acc = c->acc.as<double>();
    a.rowbits = c->rowbits.as<uint32_t>();
    a.partials = c->partials.as<long long>();
    a.acct = c->acct.as<long long>();
    a.y_idx = yi;
    a.y_val = (sr == TSMV_OR_AND) ? nullptr : yv;
    a.y_cap = ycap;
    a.ynnz_dev = ynnz_dev;
    a.cnt = c->counters.as<Counters>();
    a.hm = c->hcnt_dev;
    a.bar_base = c->bar_base;
    a.tring = c->timing ? c->tring.as<unsigned long long>() : nullptr;
    a.tslot = c->tcalls;
    void *args[] = {&a};
    void *f = pick_kernel(c->nt, f32, sr);
    TSMV_CUDA(cudaLaunchCooperativeKernel(f, dim3(c->fused_blocks), dim3(FB), args, 0, st));
    c->bar_base += 4ull * (unsigned long long)c->fused_blocks;
    if (c->timing) c->tcalls++;
}

void stats_from_partials(tsmv_ctx *c, tsmv_call_stats *s) {
    std::vector<long long> p(8 * (size_t)c->fused_blocks), q(4 * (size_t)c->fused_blocks);
    TSMV_CUDA(cudaMemcpy(p.data(), c->partials.p, p.size() * 8, cudaMemcpyDeviceToHost));
    TSMV_CUDA(cudaMemcpy(q.data(), c->acct.p, q.size() * 8, cudaMemcpyDeviceToHost));
    s->x_segments = s->tile_items = s->side_items = 0;
    s->hit_tiles = s->hit_columns = s->tile_macs = 0;
    long long nLs = 0;
    for (int b = 0; b < c->fused_blocks; ++b) {
        s->x_segments += p[8 * b];
        s->tile_items += p[8 * b + 1];
        nLs += p[8 * b + 2];
        s->side_items += p[8 * b + 3];
        s->hit_tiles += q[4 * b];
        s->hit_columns += q[4 * b + 1];
        s->tile_macs += q[4 * b + 2];
    }
    (void)nLs;
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
        c->last_x_nnz = x_nnz;
        if (x_nnz == 0) return TSMV_OK;
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
        enqueue_spmspv(c, sr, x_nnz, xi, xv, ycap_dev, yi, yv, nullptr, st);
        TSMV_CUDA(cudaStreamSynchronize(st));
        volatile Counters *h = c->hcnt;
        int64_t ynnz = h->y_nnz;
        int err = h->err;
        TSMV_REQUIRE(err == 0, "tsmv_spmspv: x indices must be strictly ascending and in [0, %lld)", (long long)c->n);
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

extern "C" tsmv_status tsmv_spmspv_async(tsmv_ctx *c, tsmv_semiring sr, int64_t x_nnz, const int32_t *x_idx,
                                         const void *x_val, int64_t y_cap, int32_t *y_idx, void *y_val,
                                         int64_t *y_nnz_dev, void *cuda_stream) {
    try {
        TSMV_REQUIRE(c != nullptr, "tsmv_spmspv_async: NULL ctx");
        TSMV_REQUIRE(sr >= 0 && sr <= 2, "tsmv_spmspv_async: bad semiring %d", (int)sr);
        TSMV_REQUIRE(x_nnz >= 1 && x_nnz <= c->n, "tsmv_spmspv_async: x_nnz %lld out of [1, ncols]",
                     (long long)x_nnz);
        TSMV_REQUIRE(x_idx != nullptr && (sr == TSMV_OR_AND || x_val != nullptr), "tsmv_spmspv_async: NULL x");
        TSMV_REQUIRE(y_cap >= 0 && (y_cap == 0 || y_idx != nullptr), "tsmv_spmspv_async: NULL y_idx");
        TSMV_REQUIRE(sr == TSMV_OR_AND || y_cap == 0 || y_val != nullptr, "tsmv_spmspv_async: NULL y_val");
        TSMV_CUDA(cudaSetDevice(c->device));
        c->last_x_nnz = x_nnz;
        enqueue_spmspv(c, sr, x_nnz, x_idx, sr == TSMV_OR_AND ? nullptr : x_val, y_cap, y_idx,
                       sr == TSMV_OR_AND ? nullptr : y_val, (long long *)y_nnz_dev, (cudaStream_t)cuda_stream);
        return TSMV_OK;
    } catch (const Err &e) {
        return e.st;
    }
}

extern "C" tsmv_status tsmv_set_timing(tsmv_ctx *c, int32_t enable) {
    try {
        TSMV_REQUIRE(c, "tsmv_set_timing: NULL ctx");
        if (enable && !c->tring.p) c->tring.alloc((size_t)TRING * 8 * 8);
        c->timing = enable != 0;
        c->tcalls = 0;
        return TSMV_OK;
    } catch (const Err &e) {
        return e.st;
    }
}

extern "C" tsmv_status tsmv_get_timing(tsmv_ctx *c, double *ms_out, int64_t *calls) {
    try {
        TSMV_REQUIRE(c && ms_out && calls, "tsmv_get_timing: NULL argument");
        for (int i = 0; i < 4; ++i) ms_out[i] = 0;
        long long n = std::min<long long>(c->tcalls, TRING);
        *calls = n;
        if (n == 0 || !c->tring.p) return TSMV_OK;
        TSMV_CUDA(cudaDeviceSynchronize());
        std::vector<unsigned long long> r((size_t)TRING * 8);
        TSMV_CUDA(cudaMemcpy(r.data(), c->tring.p, r.size() * 8, cudaMemcpyDeviceToHost));
        for (long long q = 0; q < n; ++q) {
            const unsigned long long *t = &r[q * 8];
            ms_out[0] += (t[2] - t[0]) * 1e-6;  // phase A (+A')
            ms_out[1] += (t[3] - t[2]) * 1e-6;  // phase B (expand)
            ms_out[2] += (t[5] - t[3]) * 1e-6;  // phase C (compact)
            ms_out[3] += (t[5] - t[0]) * 1e-6;  // whole kernel (block 0's view)
        }
        c->tcalls = 0;
        return TSMV_OK;
    } catch (const Err &e) {
        return e.st;
    }
}

extern "C" tsmv_status tsmv_last_call_stats(tsmv_ctx *c, tsmv_call_stats *s) {
    try {
        TSMV_REQUIRE(c && s, "tsmv_last_call_stats: NULL argument");
        TSMV_CUDA(cudaSetDevice(c->device));
        volatile Counters *h = c->hcnt;
        s->x_nnz = c->last_x_nnz;
        s->y_nnz = h->y_nnz;
        stats_from_partials(c, s);
        return TSMV_OK;
    } catch (const Err &e) {
        return e.st;
    }
}
