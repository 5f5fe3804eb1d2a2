// bfs.cu -- TileBFS (Sec 3.4 P:862-1628,
// Alg 3, Alg 5-7).
//
// State: visited bitmap V, frontier bitmaps F (current) / Fn (next), 1 bit per
// vertex, LSB-first inside uint32 words (the paper's MSB-first order, P:1458,
// is internal and does not cross the ABI -- DESIGN.md R8).  One level:
//   expand  -- Push-CSC (Alg 5): vector-driven, per frontier segment walk its
//              tile column, OR the bit planes of the frontier's columns;
//              Push-CSR (Alg 6): matrix-driven, every tile of the row-tile
//              structure whose x segment is non-empty, row words AND x word;
//              Pull-CSC (Alg 7): per row tile with unvisited rows, AND their row
//              words with the frontier words, stop at the first hit;
//              side matrix: push through its CSC / pull through
//              its CSR (the paper hands this part to GSwitch; here it is ours).
//              Discovery = atomicOr into V, new bits = bits & ~old: each vertex
//              is claimed exactly once; its level is written and its bit set in Fn.
//   scan    -- Fn -> per-segment lists + tile/side work prefixes + |F|, m_f,
//              sum indeg (one look-back pass over the n/nt segments); clears F.
// Reading R10: pull tests the frontier of the level (not the live visited
// set), so in-level discoveries cannot shorten levels.
#include "device.cuh"

namespace tsmv {

namespace {

struct Oct {
    long long v[8];
};
struct OctSum {
    __device__ __forceinline__ Oct operator()(const Oct &a, const Oct &b) const {
        Oct r;
#pragma unroll
        for (int i = 0; i < 8; ++i) r.v[i] = a.v[i] + b.v[i];
        return r;
    }
};

struct BfsView {
    uint32_t *V, *F, *Fn;
    int32_t *levels;
    long long row_begin, m_local, n;
    int level;  // level of F; discoveries get level + 1
};

template <int NT>
__device__ __forceinline__ void discover(const BfsView &B, long long gseg, typename Tr<NT>::word_t bits) {
    using word_t = typename Tr<NT>::word_t;
    word_t old = seg_or<NT>(B.V, gseg, bits);
    word_t nw = bits & ~old;
    if (nw) {
        seg_or<NT>(B.Fn, gseg, nw);
        long long base = gseg * NT - B.row_begin;
        while (nw) {
            int r = ffs_w(nw);
            nw &= nw - 1;
            B.levels[base + r] = B.level + 1;
        }
    }
}

__global__ void k_bfs_init(BfsView B, long long NW, long long source) {
    long long tid = blockIdx.x * (long long)blockDim.x + threadIdx.x;
    long long stride = (long long)gridDim.x * blockDim.x;
    for (long long w = tid; w < NW; w += stride) {
        long long v0 = w * 32;
        uint32_t pad = 0;
        if (v0 + 32 > B.n) pad = (v0 >= B.n) ? 0xffffffffu : (0xffffffffu << (B.n - v0));
        uint32_t s = (source >= v0 && source < v0 + 32) ? (1u << (source - v0)) : 0u;
        B.V[w] = pad | s;
        B.F[w] = s;
        B.Fn[w] = 0;
    }
    for (long long v = tid; v < B.m_local; v += stride)
        B.levels[v] = (v + B.row_begin == source) ? 0 : -1;
}

// Frontier scan: one thread per nt-segment of the (global) frontier bitmap F.
template <int NT>
__global__ void __launch_bounds__(SCAN_BLOCK)
k_fscan(const uint32_t *__restrict__ F, uint32_t *__restrict__ Fclear, long long nseg, long long NWpad,
        const long long *__restrict__ tptr, const long long *__restrict__ sptr, const int *__restrict__ outdeg,
        const int *__restrict__ indeg, long long row_begin, long long m_local, ListsView Lv,
        Counters *__restrict__ cnt, Counters *__restrict__ hm, LBDesc<8> *__restrict__ desc, unsigned epoch) {
    using word_t = typename Tr<NT>::word_t;
    using BS = cub::BlockScan<Oct, SCAN_BLOCK>;
    __shared__ typename BS::TempStorage ts;
    __shared__ unsigned s_bid;
    __shared__ long long s_pre[8];
    if (threadIdx.x == 0) s_bid = atomicAdd(&cnt->bid_scan, 1u);
    __syncthreads();
    const unsigned bid = s_bid;
    const long long J = (long long)bid * SCAN_BLOCK + threadIdx.x;
    Oct q;
#pragma unroll
    for (int i = 0; i < 8; ++i) q.v[i] = 0;
    word_t bits = 0;
    long long wt = 0;
    if (J < nseg) {
        bits = seg_bits<NT>(F, J);
        if (bits) {
            wt = tptr[J + 1] - tptr[J];
            q.v[0] = wt > 0;
            q.v[1] = wt;
            word_t b = bits;
            while (b) {
                int r = ffs_w(b);
                b &= b - 1;
                long long v = J * NT + r;
                long long ws = sptr[v + 1] - sptr[v];
                q.v[2] += ws > 0;
                q.v[3] += ws;
                q.v[5] += outdeg[v];
                long long lv = v - row_begin;
                if (lv >= 0 && lv < m_local) q.v[6] += indeg[lv];
            }
            q.v[4] = popc_w(bits);
        }
        // clear the consumed frontier (the level that was just expanded)
        if (Fclear) {
            if constexpr (NT == 16) {
                if ((J & 1) == 0) Fclear[J >> 1] = 0u;
            } else if constexpr (NT == 32) {
                Fclear[J] = 0u;
            } else {
                Fclear[2 * J] = 0u;
                Fclear[2 * J + 1] = 0u;
            }
        }
    }
    Oct ex, agg;
    Oct zero;
#pragma unroll
    for (int i = 0; i < 8; ++i) zero.v[i] = 0;
    BS(ts).ExclusiveScan(q, ex, zero, OctSum(), agg);
    if (threadIdx.x < 32) {
        long long pre[8];
        lookback_warp<8>(desc, bid, epoch, agg.v, pre, threadIdx.x);
        if (threadIdx.x == 0) {
#pragma unroll
            for (int i = 0; i < 8; ++i) s_pre[i] = pre[i];
        }
    }
    __syncthreads();
#pragma unroll
    for (int i = 0; i < 8; ++i) ex.v[i] += s_pre[i];
    if (bits && wt > 0) {
        long long i = ex.v[0];
        Lv.Lt_seg[i] = J;
        Lv.Lt_mask[i] = (unsigned long long)bits;
        Lv.Lt_tbeg[i] = tptr[J];
        Lv.Lt_wpre[i] = ex.v[1];
        write_chunks(Lv.Ct, ex.v[1], wt, (int)i);
    }
    if (bits) {
        long long i = ex.v[2], w0 = ex.v[3];
        word_t b = bits;
        while (b) {
            int r = ffs_w(b);
            b &= b - 1;
            long long v = J * NT + r;
            long long ws = sptr[v + 1] - sptr[v];
            if (ws > 0) {
                Lv.Ls_beg[i] = sptr[v];
                Lv.Ls_wpre[i] = w0;
                Lv.Ls_col[i] = (int)v;
                write_chunks(Lv.Cs, w0, ws, (int)i);
                ++i;
                w0 += ws;
            }
        }
    }
    if (bid == gridDim.x - 1 && threadIdx.x == SCAN_BLOCK - 1) {
        long long tot[8];
#pragma unroll
        for (int i = 0; i < 8; ++i) tot[i] = s_pre[i] + agg.v[i];
        cnt->nLt = tot[0];
        cnt->Wt = tot[1];
        cnt->nLs = tot[2];
        cnt->Ws = tot[3];
        cnt->nCt = (tot[1] + CHUNK - 1) >> CHUNK_LOG;
        cnt->nCs = (tot[3] + CHUNK - 1) >> CHUNK_LOG;
        cnt->fsize = tot[4];
        cnt->mf = tot[5];
        cnt->din = tot[6];
        Lv.Lt_wpre[tot[0]] = tot[1];
        Lv.Ls_wpre[tot[2]] = tot[3];
        hm->fsize = tot[4];
        hm->mf = tot[5];
        hm->din = tot[6];
        hm->nLt = tot[0];
        hm->Wt = tot[1];
        hm->nLs = tot[2];
        hm->Ws = tot[3];
        cnt->chunk_next = 0;
        cnt->bid_scan = 0;
    }
}

struct BfsTiles {
    const long long *ptr;
    const int *trow, *tgrp;
    const void *mask;
    const void *planes;
    long long T;
    const long long *sptr;
    const int *srow;
    const int32_t *hot_list;  // side rows of hot tile rows are encoded (TileSet::hot_list)
};

inline BfsTiles bfs_tiles(const TileSet &S) {
    BfsTiles b;
    b.ptr = S.ptr.as<long long>();
    b.trow = S.trow.as<int>();
    b.tgrp = S.tgrp.as<int>();
    b.mask = S.mask.p;
    b.planes = S.planes.p;
    b.T = S.T;
    b.sptr = S.sptr.as<long long>();
    b.srow = S.srow.as<int>();
    b.hot_list = S.hot_list;
    return b;
}

// Push (vector-driven): tile chunks (Push-CSC, Alg 5) and side chunks.
template <int NT, bool DO_TILES>
__global__ void __launch_bounds__(256)
k_push(BfsTiles P, ListsView Lv, Counters *__restrict__ cnt, BfsView B) {
    using word_t = typename Tr<NT>::word_t;
    __shared__ long long win_all[8][CHUNK + 1];
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    long long *win = win_all[wid];
    const long long nCt = DO_TILES ? cnt->nCt : 0, nCs = cnt->nCs;
    const long long nLt = cnt->nLt, nLs = cnt->nLs, Wt = cnt->Wt, Ws = cnt->Ws;
    const word_t *mask = (const word_t *)P.mask;
    const word_t *planes = (const word_t *)P.planes;
    const long long rb_seg = B.row_begin / NT;
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
                word_t hit = mask[t] & (word_t)Lv.Lt_mask[s];
                if (hit) {
                    word_t w = 0;
                    while (hit) {
                        int c = ffs_w(hit);
                        hit &= hit - 1;
                        w |= planes[(long long)c * P.T + t];
                    }
                    discover<NT>(B, rb_seg + P.trow[t], w);
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
                long long v = B.row_begin + decode_row<NT>(P.srow[p], P.hot_list);
                discover<NT>(B, v / NT, (word_t)1 << (v % NT));
            }
            __syncwarp();
        } else {
            break;
        }
    }
}

// Push-CSR (Alg 6): every tile of the row-tile structure Q; x word of its tile
// column, row words of the still-unvisited rows.
template <int NT>
__global__ void __launch_bounds__(256) k_push_csr(BfsTiles Q, BfsView B) {
    using word_t = typename Tr<NT>::word_t;
    const word_t *planes = (const word_t *)Q.planes;
    const long long rb_seg = B.row_begin / NT;
    for (long long t = blockIdx.x * (long long)blockDim.x + threadIdx.x; t < Q.T;
         t += (long long)gridDim.x * blockDim.x) {
        long long Jx = Q.trow[t];            // A's tile column (segment of x)
        word_t f = seg_bits<NT>(B.F, Jx);
        if (!f) continue;
        long long Iseg = rb_seg + Q.tgrp[t]; // A's tile row (global segment)
        word_t um = ~seg_bits<NT>(B.V, Iseg);
        if (!um) continue;
        word_t res = 0;
        while (um) {
            int r = ffs_w(um);
            um &= um - 1;
            if (planes[(long long)r * Q.T + t] & f) res |= (word_t)1 << r;
        }
        if (res) discover<NT>(B, Iseg, res);
    }
}

// Pull-CSC (Alg 7): one warp per local row tile with unvisited rows; lanes walk
// the tiles of the row tile; stop when every unvisited row has found a parent.
template <int NT>
__global__ void __launch_bounds__(256) k_pull(BfsTiles Q, BfsView B, long long nTR_local) {
    using word_t = typename Tr<NT>::word_t;
    const word_t *planes = (const word_t *)Q.planes;
    const int lane = threadIdx.x & 31;
    const long long warp = (blockIdx.x * (long long)blockDim.x + threadIdx.x) >> 5;
    const long long nwarps = ((long long)gridDim.x * blockDim.x) >> 5;
    const long long rb_seg = B.row_begin / NT;
    for (long long I = warp; I < nTR_local; I += nwarps) {
        word_t um = ~seg_bits<NT>(B.V, rb_seg + I);
        if (!um) continue;
        word_t found = 0;
        const long long t0 = Q.ptr[I], t1 = Q.ptr[I + 1];
        for (long long tb = t0; tb < t1; tb += 32) {
            long long t = tb + lane;
            word_t fl = 0;
            if (t < t1) {
                word_t f = seg_bits<NT>(B.F, Q.trow[t]);
                if (f) {
                    word_t u = um;
                    while (u) {
                        int r = ffs_w(u);
                        u &= u - 1;
                        if (planes[(long long)r * Q.T + t] & f) fl |= (word_t)1 << r;
                    }
                }
            }
            fl = warp_or(fl);
            found |= fl;
            um &= ~fl;
            if (!um) break;
        }
        if (lane == 0 && found) discover<NT>(B, rb_seg + I, found);
    }
}

// Pull over the side matrix: CSC of A^T's side part = in-neighbour lists.
template <int NT>
__global__ void __launch_bounds__(256) k_pull_side(BfsTiles Q, BfsView B) {
    using word_t = typename Tr<NT>::word_t;
    for (long long v = blockIdx.x * (long long)blockDim.x + threadIdx.x; v < B.m_local;
         v += (long long)gridDim.x * blockDim.x) {
        long long p0 = Q.sptr[v], p1 = Q.sptr[v + 1];
        if (p0 == p1) continue;
        long long g = B.row_begin + v;
        if ((B.V[g >> 5] >> (g & 31)) & 1u) continue;
        for (long long p = p0; p < p1; ++p) {
            long long u = decode_row<NT>(Q.srow[p], Q.hot_list);
            if ((B.F[u >> 5] >> (u & 31)) & 1u) {
                discover<NT>(B, g / NT, (word_t)1 << (g % NT));
                break;
            }
        }
    }
}

__global__ void k_merge(const uint32_t *__restrict__ gathered, long long stride, int nranks,
                        const long long *__restrict__ splits, int self, uint32_t *__restrict__ Fn,
                        uint32_t *__restrict__ V) {
    for (int p = 0; p < nranks; ++p) {
        if (p == self) continue;
        long long w0 = splits[p] >> 5;
        long long nw = (splits[p + 1] - splits[p] + 31) >> 5;
        for (long long w = blockIdx.x * (long long)blockDim.x + threadIdx.x; w < nw;
             w += (long long)gridDim.x * blockDim.x) {
            uint32_t b = gathered[p * stride + w];
            if (b) {
                Fn[w0 + w] |= b;
                V[w0 + w] |= b;
            }
        }
    }
}

inline int grid_for(long long n, int bs = 256, int maxg = 148 * 16) {
    long long g = (n + bs - 1) / bs;
    if (g < 1) g = 1;
    if (g > maxg) g = maxg;
    return (int)g;
}

}  // namespace

// ----------------------------------------------------------------- host side
struct BfsRunner {
    tsmv_ctx *c;
    cudaStream_t st;
    long long NW;

    BfsView view() {
        BfsView B;
        B.V = c->V.as<uint32_t>();
        B.F = (c->fcur == 0 ? c->F0 : c->F1).as<uint32_t>();
        B.Fn = (c->fcur == 0 ? c->F1 : c->F0).as<uint32_t>();
        B.levels = c->levels_dev;
        B.row_begin = c->row_begin;
        B.m_local = c->m;
        B.n = c->n;
        B.level = c->bfs_level;
        return B;
    }

    template <int NT> void fscan(const uint32_t *F, uint32_t *Fclear) {
        long long nseg = c->nTC;
        int grid = (int)std::max<long long>(1, (nseg + SCAN_BLOCK - 1) / SCAN_BLOCK);
        c->epoch++;
        k_fscan<NT><<<grid, SCAN_BLOCK, 0, st>>>(F, Fclear, nseg, NW, c->P.ptr.as<long long>(),
                                                 c->P.sptr.as<long long>(), c->outdeg.as<int>(), c->indeg.as<int>(),
                                                 c->row_begin, c->m, lists_view(c), c->counters.as<Counters>(),
                                                 c->hcnt_dev, c->desc_bfs.as<LBDesc<8>>(), c->epoch);
        TSMV_CUDA(cudaGetLastError());
    }

    template <int NT> void expand(int dir) {
        BfsView B = view();
        BfsTiles P = bfs_tiles(c->P), Q = bfs_tiles(*c->Q);
        if (dir == TSMV_DIR_PUSH_CSC) {
            k_push<NT, true><<<c->expand_blocks, 256, 0, st>>>(P, lists_view(c), c->counters.as<Counters>(), B);
        } else if (dir == TSMV_DIR_PUSH_CSR) {
            k_push<NT, false><<<c->expand_blocks, 256, 0, st>>>(P, lists_view(c), c->counters.as<Counters>(), B);
            if (Q.T) k_push_csr<NT><<<grid_for(Q.T), 256, 0, st>>>(Q, B);
        } else {
            long long nTRl = (c->m + NT - 1) / NT;
            k_pull<NT><<<grid_for(nTRl * 32), 256, 0, st>>>(Q, B, nTRl);
            k_pull_side<NT><<<grid_for(c->m), 256, 0, st>>>(Q, B);
        }
        TSMV_CUDA(cudaGetLastError());
    }

    void do_fscan(const uint32_t *F, uint32_t *Fclear) {
        switch (c->nt) {
            case 16: fscan<16>(F, Fclear); break;
            case 32: fscan<32>(F, Fclear); break;
            default: fscan<64>(F, Fclear); break;
        }
    }
    void do_expand(int dir) {
        switch (c->nt) {
            case 16: expand<16>(dir); break;
            case 32: expand<32>(dir); break;
            default: expand<64>(dir); break;
        }
    }
    void init(long long source) {
        BfsView B = view();
        k_bfs_init<<<grid_for(std::max<long long>(NW, c->m)), 256, 0, st>>>(B, NW, source);
        TSMV_CUDA(cudaGetLastError());
    }
};

int choose_dir(const tsmv_options &o, long long n, long long fsize, long long mf, long long mu) {
    if (o.force_dir != TSMV_DIR_AUTO) return o.force_dir;
    // reading R9: Beamer-style edge test for pull, then the paper's 0.01 density rule
    if ((double)mf > (double)mu / o.pull_alpha) return TSMV_DIR_PULL_CSC;
    if ((double)fsize / (double)n >= o.push_csr_density) return TSMV_DIR_PUSH_CSR;
    return TSMV_DIR_PUSH_CSC;
}

}  // namespace tsmv

using namespace tsmv;

static void bfs_check(tsmv_ctx *c) {
    TSMV_REQUIRE(c->bfs_built, "tsmv_bfs: context built without BFS structures (square A and build_bfs=1 needed)");
}

static void bfs_prepare_levels(tsmv_ctx *c, int32_t *levels, bool &host_levels) {
    host_levels = !is_device_ptr(levels);
    if (host_levels) {
        c->stage_levels.ensure(std::max<int64_t>(c->m, 1) * 4);
        c->levels_dev = c->stage_levels.as<int32_t>();
    } else {
        c->levels_dev = levels;
    }
}

extern "C" tsmv_status tsmv_bfs(tsmv_ctx *c, int64_t source, int32_t *levels, tsmv_bfs_stats *stats,
                                void *cuda_stream) {
    try {
        TSMV_REQUIRE(c != nullptr && levels != nullptr, "tsmv_bfs: NULL argument");
        bfs_check(c);
        TSMV_REQUIRE(c->opt.nranks == 1, "tsmv_bfs: distributed contexts use tsmv_bfs_dist_*");
        TSMV_REQUIRE(source >= 0 && source < c->n, "tsmv_bfs: source %lld out of range", (long long)source);
        TSMV_CUDA(cudaSetDevice(c->device));
        cudaStream_t st = (cudaStream_t)cuda_stream;
        bool host_levels;
        bfs_prepare_levels(c, levels, host_levels);
        ensure_lists(c, c->n);
        BfsRunner R{c, st, (long long)(c->V.bytes / 4)};
        c->fcur = 0;
        c->bfs_level = 0;
        TSMV_CUDA(cudaEventRecord(c->ev0, st));
        R.init(source);
        R.do_fscan(c->F0.as<uint32_t>(), nullptr);
        TSMV_CUDA(cudaStreamSynchronize(st));
        volatile Counters *h = c->hcnt;
        long long fsize = h->fsize, mf = h->mf;
        long long mu = c->nnz - h->din;
        long long reached = 0, edges = 0;
        int L = 0;
        if (stats) stats->nlevels = 0;
        while (fsize > 0) {
            int dir = choose_dir(c->opt, c->n, fsize, mf, mu);
            if (stats && L < TSMV_MAX_LEVELS) {
                stats->dir_per_level[L] = dir;
                stats->frontier_per_level[L] = fsize;
            }
            reached += fsize;
            edges += mf;
            c->bfs_level = L;
            R.do_expand(dir);
            uint32_t *Fcur = (c->fcur == 0 ? c->F0 : c->F1).as<uint32_t>();
            uint32_t *Fnext = (c->fcur == 0 ? c->F1 : c->F0).as<uint32_t>();
            R.do_fscan(Fnext, Fcur);
            TSMV_CUDA(cudaStreamSynchronize(st));
            fsize = h->fsize;
            mf = h->mf;
            mu -= h->din;
            c->fcur ^= 1;
            ++L;
        }
        TSMV_CUDA(cudaEventRecord(c->ev1, st));
        // leave F clean for the next traversal
        TSMV_CUDA(cudaMemsetAsync(c->F0.p, 0, c->F0.bytes, st));
        TSMV_CUDA(cudaMemsetAsync(c->F1.p, 0, c->F1.bytes, st));
        if (host_levels) TSMV_CUDA(cudaMemcpyAsync(levels, c->levels_dev, c->m * 4, cudaMemcpyDeviceToHost, st));
        TSMV_CUDA(cudaStreamSynchronize(st));
        if (stats) {
            float ms = 0;
            TSMV_CUDA(cudaEventElapsedTime(&ms, c->ev0, c->ev1));
            stats->nlevels = L;
            stats->reached = reached;
            stats->edges_traversed = edges;
            stats->ms = ms;
        }
        return TSMV_OK;
    } catch (const Err &e) {
        return e.st;
    }
}

// ----------------------------------------------------------------- distributed primitives
extern "C" int64_t tsmv_owned_words(const tsmv_ctx *c) { return c ? (c->m + 31) / 32 : 0; }

extern "C" tsmv_status tsmv_bfs_dist_begin(tsmv_ctx *c, int64_t source, int32_t *levels, int64_t *out_stats,
                                           void *cuda_stream) {
    try {
        TSMV_REQUIRE(c && levels && out_stats, "tsmv_bfs_dist_begin: NULL argument");
        bfs_check(c);
        TSMV_REQUIRE(source >= 0 && source < c->n, "tsmv_bfs_dist_begin: source out of range");
        TSMV_REQUIRE(is_device_ptr(levels), "tsmv_bfs_dist_begin: levels must be device memory");
        TSMV_CUDA(cudaSetDevice(c->device));
        cudaStream_t st = (cudaStream_t)cuda_stream;
        c->levels_dev = levels;
        ensure_lists(c, c->n);
        BfsRunner R{c, st, (long long)(c->V.bytes / 4)};
        c->fcur = 0;
        c->bfs_level = 0;
        TSMV_CUDA(cudaMemsetAsync(c->F1.p, 0, c->F1.bytes, st));
        R.init(source);
        R.do_fscan(c->F0.as<uint32_t>(), nullptr);
        TSMV_CUDA(cudaStreamSynchronize(st));
        volatile Counters *h = c->hcnt;
        c->m_u_local = c->nnz - h->din;
        out_stats[0] = h->fsize;
        out_stats[1] = h->mf;
        out_stats[2] = c->m_u_local;
        return TSMV_OK;
    } catch (const Err &e) {
        return e.st;
    }
}

extern "C" tsmv_status tsmv_bfs_dist_expand(tsmv_ctx *c, int32_t dir, uint32_t *owned_words_out, void *cuda_stream) {
    try {
        TSMV_REQUIRE(c && owned_words_out, "tsmv_bfs_dist_expand: NULL argument");
        TSMV_REQUIRE(dir >= 1 && dir <= 3, "tsmv_bfs_dist_expand: dir must be concrete (1..3)");
        TSMV_CUDA(cudaSetDevice(c->device));
        cudaStream_t st = (cudaStream_t)cuda_stream;
        BfsRunner R{c, st, (long long)(c->V.bytes / 4)};
        R.do_expand(dir);
        uint32_t *Fnext = (c->fcur == 0 ? c->F1 : c->F0).as<uint32_t>();
        TSMV_CUDA(cudaMemcpyAsync(owned_words_out, Fnext + (c->row_begin >> 5), tsmv_owned_words(c) * 4,
                                  cudaMemcpyDeviceToDevice, st));
        return TSMV_OK;
    } catch (const Err &e) {
        return e.st;
    }
}

extern "C" tsmv_status tsmv_bfs_dist_merge(tsmv_ctx *c, const uint32_t *gathered, int64_t stride_words,
                                           int64_t *out_stats, void *cuda_stream) {
    try {
        TSMV_REQUIRE(c && out_stats, "tsmv_bfs_dist_merge: NULL argument");
        TSMV_CUDA(cudaSetDevice(c->device));
        cudaStream_t st = (cudaStream_t)cuda_stream;
        BfsRunner R{c, st, (long long)(c->V.bytes / 4)};
        uint32_t *Fcur = (c->fcur == 0 ? c->F0 : c->F1).as<uint32_t>();
        uint32_t *Fnext = (c->fcur == 0 ? c->F1 : c->F0).as<uint32_t>();
        if (c->opt.nranks > 1) {
            TSMV_REQUIRE(gathered != nullptr, "tsmv_bfs_dist_merge: NULL gathered");
            k_merge<<<grid_for(stride_words), 256, 0, st>>>(gathered, stride_words, c->opt.nranks,
                                                            c->splits_dev.as<long long>(), c->opt.rank, Fnext,
                                                            c->V.as<uint32_t>());
            TSMV_CUDA(cudaGetLastError());
        }
        R.do_fscan(Fnext, Fcur);
        TSMV_CUDA(cudaStreamSynchronize(st));
        volatile Counters *h = c->hcnt;
        c->m_u_local -= h->din;
        c->fcur ^= 1;
        c->bfs_level += 1;
        out_stats[0] = h->fsize;
        out_stats[1] = h->mf;
        out_stats[2] = c->m_u_local;
        return TSMV_OK;
    } catch (const Err &e) {
        return e.st;
    }
}

extern "C" int32_t tsmv_choose_dir(const tsmv_options *o, int64_t n, int64_t frontier, int64_t m_f, int64_t m_u) {
    tsmv_options d;
    if (!o) {
        tsmv_default_options(&d);
        o = &d;
    }
    return choose_dir(*o, n, frontier, m_f, m_u);
}
