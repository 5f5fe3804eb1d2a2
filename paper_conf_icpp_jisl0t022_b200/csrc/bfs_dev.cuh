// bfs_dev.cuh -- device-side pieces of one TileBFS level shared by the
// per-level kernels (bfs.cu, used by the distributed driver) and the fused
// persistent single-GPU kernel (bfs_fused.cu).
#pragma once
#include "device.cuh"

namespace tsmv {

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

struct BfsTiles {
    const long long *ptr;
    const int *trow, *tgrp;
    const void *mask;
    const void *planes;
    long long T;
    const long long *sptr;
    const int *srow;
    const int32_t *hot_list;  // side rows of hot tile rows are encoded (TileSet::hot_list)
    const unsigned long long *pmask;  // per group: planes with a nonzero (rows the tile part can discover)
    const uint32_t *smask;            // per 32 columns: side columns with a nonzero (rows the side part can discover)
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
    b.pmask = S.pmask.as<unsigned long long>();
    b.smask = S.smask.as<uint32_t>();
    return b;
}


// ---- one item of each level kernel -------------------------------------------

// heavy Push-CSC level of the per-level kernels (push items > rows / 8): bulk mode
__host__ __device__ __forceinline__ bool push_bulk(bool csc, long long Wt, long long Ws, long long rows) {
    return csc && (Wt + Ws) * 8 > rows;
}

// Bulk push (r2): the rows reached are only ORed into the next-frontier bitmap
// with fire-and-forget reductions; a pass over the words afterwards takes new =
// Fn & ~V, sets V and the levels (heavy Push-CSC levels: one returning atomic per
// edge was the bound).
template <int NT>
__device__ __forceinline__ void reach(const BfsView &B, long long gseg, typename Tr<NT>::word_t bits, bool bulk) {
    if (bulk) (void)seg_or<NT>(B.Fn, gseg, bits);
    else discover<NT>(B, gseg, bits);
}

// Push-CSC tile item (Alg 5): OR the bit planes of the frontier's columns of tile t.
template <int NT>
__device__ __forceinline__ void push_tile_item(const BfsTiles &P, const BfsView &B, long long t,
                                               typename Tr<NT>::word_t xm, bool bulk = false) {
    using word_t = typename Tr<NT>::word_t;
    word_t hit = ((const word_t *)P.mask)[t] & xm;
    if (hit) {
        const word_t *planes = (const word_t *)P.planes;
        word_t w = 0;
        while (hit) {
            int c = ffs_w(hit);
            hit &= hit - 1;
            w |= planes[(long long)c * P.T + t];
        }
        reach<NT>(B, B.row_begin / NT + P.trow[t], w, bulk);
    }
}

// Push over the side matrix: one side nonzero p of a frontier vertex's column.
template <int NT>
__device__ __forceinline__ void push_side_item(const BfsTiles &P, const BfsView &B, long long p, bool bulk = false) {
    using word_t = typename Tr<NT>::word_t;
    long long v = B.row_begin + decode_row<NT>(P.srow[p], P.hot_list);
    reach<NT>(B, v / NT, (word_t)1 << (v % NT), bulk);
}

// Rows r of `um` whose row word in tile t meets the frontier word f.  nt = 16:
// all 16 candidate plane words are loaded at once (predicated, independent),
// instead of one dependent loop trip per row.
template <int NT>
__device__ __forceinline__ typename Tr<NT>::word_t rows_hit(const typename Tr<NT>::word_t *planes, long long T,
                                                            long long t, typename Tr<NT>::word_t um,
                                                            typename Tr<NT>::word_t f) {
    using word_t = typename Tr<NT>::word_t;
    word_t res = 0;
    if constexpr (NT == 16) {
        if (__popc((unsigned)um) <= 2) {  // few candidate rows (late pull levels): plain loop
            while (um) {
                const int r = ffs_w(um);
                um &= um - 1;
                if (planes[(long long)r * T + t] & f) res |= (word_t)1 << r;
            }
            return res;
        }
        word_t w[16];
#pragma unroll
        for (int r = 0; r < 16; ++r) w[r] = ((um >> r) & 1u) ? planes[(long long)r * T + t] : (word_t)0;
#pragma unroll
        for (int r = 0; r < 16; ++r)
            if (w[r] & f) res |= (word_t)1 << r;
    } else {
        while (um) {
            int r = ffs_w(um);
            um &= um - 1;
            if (planes[(long long)r * T + t] & f) res |= (word_t)1 << r;
        }
    }
    return res;
}

// Push-CSR (Alg 6) tile item: tile t of the row structure Q; x word of its tile
// column, row words of the still-unvisited rows.
template <int NT>
__device__ __forceinline__ void push_csr_item(const BfsTiles &Q, const BfsView &B, long long t) {
    using word_t = typename Tr<NT>::word_t;
    const word_t *planes = (const word_t *)Q.planes;
    long long Jx = Q.trow[t];  // A's tile column (segment of x)
    word_t f = seg_bits<NT>(B.F, Jx);
    if (!f) return;
    long long Iseg = B.row_begin / NT + Q.tgrp[t];  // A's tile row (global segment)
    word_t um = ~seg_bits<NT>(B.V, Iseg);
    if (!um) return;
    const word_t res = rows_hit<NT>(planes, Q.T, t, um, f);
    if (res) discover<NT>(B, Iseg, res);
}

// Pull-CSC (Alg 7), one warp on local row tile I: lanes walk the tiles of the
// row tile; stop when every unvisited row has found a parent in the frontier.
template <int NT>
__device__ __forceinline__ void pull_rowtile(const BfsTiles &Q, const BfsView &B, long long I, int lane) {
    using word_t = typename Tr<NT>::word_t;
    const word_t *planes = (const word_t *)Q.planes;
    const long long rb_seg = B.row_begin / NT;
    // rows without in-edges in the tile part (isolated, or side-only) can never be
    // found here: leave them out, or they would defeat the early exit every level
    word_t um = ~seg_bits<NT>(B.V, rb_seg + I) & (word_t)Q.pmask[I];
    if (!um) return;
    word_t found = 0;
    const long long t0 = Q.ptr[I], t1 = Q.ptr[I + 1];
    for (long long tb = t0; tb < t1; tb += 32) {
        long long t = tb + lane;
        word_t fl = 0;
        if (t < t1) {
            word_t f = seg_bits<NT>(B.F, Q.trow[t]);
            if (f) fl = rows_hit<NT>(planes, Q.T, t, um, f);
        }
        fl = warp_or(fl);
        found |= fl;
        um &= ~fl;
        if (!um) break;
    }
    if (lane == 0 && found) discover<NT>(B, rb_seg + I, found);
}

// Pull-CSC over 32 consecutive row tiles I0 .. I0+31 with one warp: the lanes
// test the visited words of all 32 in one coalesced load, and only the row
// tiles that still have unvisited rows are walked (pull_rowtile), one by one.
template <int NT>
__device__ __forceinline__ void pull_rowtiles32(const BfsTiles &Q, const BfsView &B, long long I0, long long nTR,
                                                int lane) {
    using word_t = typename Tr<NT>::word_t;
    const long long I = I0 + lane;
    bool open = false;
    if (I < nTR) open = ((word_t)~seg_bits<NT>(B.V, B.row_begin / NT + I) & (word_t)Q.pmask[I]) != 0;
    unsigned todo = __ballot_sync(0xffffffffu, open);
    while (todo) {
        const int l = __ffs(todo) - 1;
        todo &= todo - 1;
        pull_rowtile<NT>(Q, B, I0 + l, lane);
    }
}

// Pull over the side matrix: in-neighbour list of local vertex v (CSC of A^T's side).
// The visited bit is tested first (one coalesced word per 32 vertices), so a
// visited vertex costs no read of the side structure.
template <int NT>
__device__ __forceinline__ void pull_side_vertex(const BfsTiles &Q, const BfsView &B, long long v) {
    using word_t = typename Tr<NT>::word_t;
    long long g = B.row_begin + v;
    if ((B.V[g >> 5] >> (g & 31)) & 1u) return;
    if (!((Q.smask[v >> 5] >> (v & 31)) & 1u)) return;  // no side in-edges
    long long p0 = Q.sptr[v], p1 = Q.sptr[v + 1];
    // PR in-neighbours per round: their ids, then their frontier bits, each
    // step as independent loads (early exit between rounds)
#ifndef TSMV_PULL_ROUND
#define TSMV_PULL_ROUND 2  // r2: 2 beats 4 and 8 (R-MAT s26 480 -> 493 GTEPS, s22 314 -> 319)
#endif
    constexpr int PR = TSMV_PULL_ROUND;
    for (long long p = p0; p < p1; p += PR) {
        int sr[PR];
#pragma unroll
        for (int j = 0; j < PR; ++j) sr[j] = p + j < p1 ? Q.srow[p + j] : 0;
        bool hit = false;
#pragma unroll
        for (int j = 0; j < PR; ++j) {
            if (p + j < p1) {
                const long long u = decode_row<NT>(sr[j], Q.hot_list);
                hit |= ((B.F[u >> 5] >> (u & 31)) & 1u) != 0;
            }
        }
        if (hit) {
            discover<NT>(B, g / NT, (word_t)1 << (g % NT));
            break;
        }
    }
}

// Pull over the side matrix for the 32 vertices of visited word w (global word
// index; only vertices in [row_begin, row_begin + m_local) are local).  Used by
// the persistent kernel, whose few threads would otherwise walk the vertices
// one by one: a fully visited word costs one load.
template <int NT>
__device__ __forceinline__ void pull_side_word(const BfsTiles &Q, const BfsView &B, long long w) {
    const long long wl = w - B.row_begin / 32;  // local word (row_begin is a multiple of 64)
    uint32_t um = ~B.V[w] & Q.smask[wl];
    while (um) {
        const int r = __ffs(um) - 1;
        um &= um - 1;
        const long long v = w * 32 + r - B.row_begin;
        if (v < 0 || v >= B.m_local) continue;
        pull_side_vertex<NT>(Q, B, v);
    }
}

// Device copy of the direction rule (reading R9); host: tsmv::choose_dir.
__device__ __forceinline__ int choose_dir_dev(int force, double alpha, double dens, long long n, long long f,
                                              long long mf, long long mu, double alpha_burst = 0,
                                              double growth = 0, long long fprev = 0) {
    if (force) return force;
    if ((double)mf > (double)mu / burst_alpha(alpha, alpha_burst, growth, f, fprev)) return TSMV_DIR_PULL_CSC;
    if ((double)f / (double)n >= dens) return TSMV_DIR_PUSH_CSR;
    return TSMV_DIR_PUSH_CSC;
}

}  // namespace tsmv
