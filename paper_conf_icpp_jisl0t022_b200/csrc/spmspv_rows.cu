// spmspv_rows.cu -- row-driven TileSpMSpV (Alg 4, Sec 3.3
// P:790-863; SURVEY §8(a) a3 "row-driven variant: per row tile, test
// x_ptr[tile_col] != -1").  nt = 16 contexts.
//
// The column-driven flat kernel (spmspv_flat.cu) visits only the tile columns of
// x's segments but pays an L2 atomic per useful nonzero; the paper's Alg 4 walks
// the tiles of every row tile instead and skips a tile whose x segment is empty
// (here: whose column mask misses the segment's bits), so the rows of a tile row
// are summed in on-chip memory and written once, without atomics.  That pays
// when x is dense enough that most tile columns are hit anyway, and on regular
// matrices (stencils, bands: many nonzeros per tile, few very sparse tiles).
// tsmv_spmspv picks the kernel per call ("density switch").
//
// One cooperative launch, phases:
//   A  (a2) x validated and scattered into the dense x_d and the x bitmap (the
//      tiled vector: bits of segment J = x's mask of tile column J)
//   -- grid barrier -- (an invalid x leaves every workspace clean)
//   B  (a5) the side matrix (very sparse tiles, CSC) merged column-wise for x's
//      columns, warp-level balanced over the warp's x entries;
//   -- grid barrier --
//   B' (a3, a4) warp w walks its row-tile-aligned range of the row-major tile
//      list in rounds of 32 tiles (lane = tile; the next round's tile metadata and
//      x-segment bits are loaded while this round multiplies): hit = column mask
//      & x bits of the tile column, hit tiles multiplied from their 64-byte record
//      (+ index / value arrays) into a 32-slot ring of row-tile accumulators in
//      shared memory; a completed row tile is combined with the side part in acc
//      by ONE coalesced read-modify-write of its 16 rows (the warp owns the row
//      tile: no atomics), first touches counted exactly
//   -- grid barrier --
//   C  (a6) compaction (emit_pieces, shared with the flat kernel)
#include "spmspv_common.cuh"
#include <cub/device/device_radix_sort.cuh>
#include <algorithm>
#include <vector>

namespace tsmv {

namespace {

#ifndef TSMV_RT
#define TSMV_RT 512
#endif
constexpr int RT = TSMV_RT;        // threads per CTA (one CTA per SM: 128 registers at 512)
constexpr int RNW = RT / 32;       // warps per CTA
constexpr int RING = 32;           // row-tile accumulator slots per warp (>= row tiles of a 32-tile round)
constexpr int RKP = 8;             // bitmap pieces per CTA in phase C
constexpr int RMAXG = 256;
constexpr int RSPW = 4, RBATCH = 4;

struct RowArgs {
    const int32_t *x_idx;
    const void *x_val;
    long long k, n, m, W, row_begin;
    const int32_t *rrow, *rJ, *rid;  // row-major tile order: tile row, tile column, tile id in P
    const uint16_t *rmask;
    const long long *wstart;          // [G * RNW + 1]: first row-major tile of each warp's range
    const TileRec64 *rec;
    const uint8_t *idx;
    const void *val;
    const long long *sptr;
    const int *srow;
    const void *sval;
    const int32_t *hot_list;
    int n_hot;
    double *xd;
    uint32_t *xbits;
    double *acc;
    uint32_t *rowbits;
    unsigned *pc, *pc_next;
    int ps_log, n_pieces;
    int32_t *y_idx;
    void *y_val;
    long long y_cap;
    long long *ynnz_dev;
    long long *partials, *acct;
    Counters *cnt, *hm;
    unsigned long long bar_base;
};

__device__ __forceinline__ void touch_row(const RowArgs &a, unsigned *s_pc, long long row) {
    atomicOr(&a.rowbits[row >> 5], 1u << (row & 31));
    atomicAdd(&s_pc[(row >> 5) >> a.ps_log], 1u);
}

// 16 x bits of tile column J (segment J of the x bitmap)
__device__ __forceinline__ unsigned xseg(const uint32_t *xb, long long J) {
    return (__ldcg(&xb[J >> 1]) >> ((J & 1) * 16)) & 0xffffu;
}

// add a row tile's sum of row `row` (never -0.0, see prod_nz) to acc; true if
// it is the row's first contribution of the call
template <int SR>
__device__ __forceinline__ bool acc_combine(double *acc, long long row, double v) {
    if constexpr (SR == TSMV_PLUS_TIMES) {
        return (unsigned long long)__double_as_longlong(atomicAdd(&acc[row], v)) == EMPTY;
    } else if constexpr (SR == TSMV_MIN_SECOND) {
        return (unsigned long long)atomicMax((long long *)&acc[row], (long long)__double_as_longlong(v)) == EMPTY;
    } else {
        return atomicExch((unsigned long long *)&acc[row], 0ull) == EMPTY;
    }
}

template <class AV, int SR>
__device__ __forceinline__ void ring_add(double *slot16, unsigned *tmask, int r, double a, double x) {
    acc_shared<SR>(slot16, r, a, x);
    atomicOr(tmask, 1u << r);
}

template <class AV, class XV, int SR>
__global__ void __launch_bounds__(RT, 1) k_spmspv_rows(RowArgs a) {
    constexpr int NT = 16;
    __shared__ long long s_scan[8][RNW];
    __shared__ long long s_pbase[RKP], s_ex0[RKP], s_tot[4];
    __shared__ int s_nd, s_err;
    __shared__ int s_hlist[HOT_SLOTS / 16];
    __shared__ long long s_acct[RNW][4];
    __shared__ long long s_rtI[RNW][RING];  // row tile of each ring slot of the current round
    extern __shared__ __align__(16) unsigned char s_dyn[];
    double *s_ys = reinterpret_cast<double *>(s_dyn);                       // [RNW][RING][16]
    unsigned *s_yt = reinterpret_cast<unsigned *>(s_ys + RNW * RING * 16);  // [RNW][RING] touched rows
    unsigned *s_pcnt = s_yt + RNW * RING;                                   // [RMAXG * RKP]
    const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
    const int G = gridDim.x, b = blockIdx.x;
    unsigned long long target = a.bar_base;
    for (int i = tid; i < a.n_pieces; i += RT) s_pcnt[i] = 0u;
    for (int i = tid; i < a.n_hot; i += RT) s_hlist[i] = a.hot_list[i];
    for (int i = tid; i < RNW * RING * 16; i += RT) s_ys[i] = __longlong_as_double((long long)EMPTY);
    for (int i = tid; i < RNW * RING; i += RT) s_yt[i] = 0u;
    if (tid < RKP && b + tid * G < a.n_pieces) a.pc_next[b + tid * G] = 0u;
    if (tid == 0) s_err = 0;
    __syncthreads();
    long long n_seg = 0, n_tiles = 0, n_sent = 0, n_side = 0, n_hit = 0, n_hcol = 0, n_mac = 0, n_ind = 0;

    // ---------------------------------------------------------------- phase A (a2)
    const long long gw = (long long)b * RNW + wid, nwarps = (long long)G * RNW;
    for (long long e = (long long)b * RT + tid; e < a.k; e += (long long)G * RT) {
        const long long j = a.x_idx[e];
        const long long prev = e > 0 ? (long long)a.x_idx[e - 1] : -1;
        if (j < 0 || j >= a.n || prev >= j) {
            s_err = 1;
            continue;
        }
        a.xd[j] = a.x_val ? (double)((const XV *)a.x_val)[e] : 1.0;
        atomicOr(&a.xbits[j >> 5], 1u << (j & 31));
        n_seg += (e == 0 || (prev >> 4) != (j >> 4));
    }
    __syncthreads();
    if (tid == 0 && s_err) a.cnt->err = 1;
    grid_sync_f(&a.cnt->bar, target, nullptr);
    const bool err = __ldcg(&a.cnt->err) != 0;

    // ---------------------------------------------------------------- phase B (a5)
    // warp w takes x entries [32 w', 32 w' + 32) round-robin; lane = entry; the
    // warp's side columns as one list: lane = item, entry by binary search over
    // the inclusive prefix of the lengths (shuffles)
    if (!err) {
        for (long long e0 = gw * 32; e0 < a.k; e0 += nwarps * 32) {
            const long long e = e0 + lane;
            long long sb = 0, sl = 0;
            double xj = 0.0;
            if (e < a.k) {
                const long long j = a.x_idx[e];
                xj = a.x_val ? (double)((const XV *)a.x_val)[e] : 1.0;
                sb = a.sptr[j];
                sl = a.sptr[j + 1] - sb;
            }
            long long incl = sl;
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                const long long v = __shfl_up_sync(0xffffffffu, incl, o);
                if (lane >= o) incl += v;
            }
            const long long tot = __shfl_sync(0xffffffffu, incl, 31);
            n_sent += sl > 0;
            n_side += sl;
            for (long long q0 = 0; q0 < tot; q0 += 32) {
                const long long q = q0 + lane;
                int lo = 0;
#pragma unroll
                for (int step = 16; step >= 1; step >>= 1) {
                    const long long v = __shfl_sync(0xffffffffu, incl, lo + step - 1);
                    if (v <= q) lo += step;
                }
                lo = min(lo, 31);
                const long long ex = __shfl_sync(0xffffffffu, incl - sl, lo);
                const long long sbe = __shfl_sync(0xffffffffu, sb, lo);
                const double xe = __shfl_sync(0xffffffffu, xj, lo);
                if (q < tot) {
                    const long long p = sbe + (q - ex);
                    const int rc = a.srow[p];
                    const long long row = rc >= 0 ? (long long)rc : (long long)s_hlist[(~rc) / NT] * NT + ((~rc) % NT);
                    const double av = a.sval ? (double)((const AV *)a.sval)[p] : 1.0;
                    if (acc_first<SR>(a.acc, row, av, xe)) touch_row(a, s_pcnt, row);
                }
            }
        }
    }

    grid_sync_f(&a.cnt->bar, target, nullptr);

    // ---------------------------------------------------------------- phase B' (a3, a4)
    if (!err) {
        double *ys = s_ys + wid * RING * 16;
        unsigned *yt = s_yt + wid * RING;
        const long long t0 = a.wstart[gw], t1 = a.wstart[gw + 1];
        n_tiles = t1 - t0;
        // Round r covers tiles [t, t + 32).  Its distinct row tiles (ascending along
        // the lanes) take ring slots 0, 1, ... in order; the row tile carried over
        // from the previous round (its first one, if it continued) keeps slot 0.
        constexpr int INL = 32 / (int)sizeof(AV);
        long long t = t0;
        long long *rtI = s_rtI[wid];
        const unsigned lt_mask = (1u << lane) - 1u;
        // round-0 metadata
        long long I = -1, J = 0, tileid = 0;
        unsigned mk = 0, xsg = 0;
        if (t + lane < t1) {
            I = a.rrow[t + lane];
            J = a.rJ[t + lane];
            mk = a.rmask[t + lane];
            tileid = a.rid[t + lane];
        }
        if (I >= 0) xsg = xseg(a.xbits, J);
        while (t < t1) {
            // next round's metadata, in flight while this round multiplies
            const long long tn = t + 32 + lane;
            long long In = -1, Jn = 0, idn = 0;
            unsigned mkn = 0;
            if (tn < t1) {
                In = a.rrow[tn];
                Jn = a.rJ[tn];
                mkn = a.rmask[tn];
                idn = a.rid[tn];
            }
            // ring slot = ordinal of the lane's row tile among the round's row tiles
            const long long Iup = __shfl_up_sync(0xffffffffu, I, 1);
            const bool head = I >= 0 && (lane == 0 || Iup != I);
            const unsigned heads = __ballot_sync(0xffffffffu, head);
            const int ord = __popc(heads & (lt_mask | (1u << lane))) - 1;
            if (head) rtI[ord] = I;
            __syncwarp();
            const unsigned hit = I >= 0 ? (mk & xsg) : 0u;
            // hit tiles: one 64-byte record each; the useful nonzeros of the round's
            // hit tiles are then dealt over the lanes (one load of each nonzero's
            // value, index and x value per lane, all in flight together), as in the
            // flat kernel's phase B2
            unsigned off = 0, nnz = 0;
            uint4 h1 = make_uint4(0, 0, 0, 0), v0 = make_uint4(0, 0, 0, 0), v1 = make_uint4(0, 0, 0, 0);
            int useful = 0;
            if (hit) {
                uint4 h0;
                ld32_nc(a.rec + tileid, h0, h1);
                ld32_nc(reinterpret_cast<const uint4 *>(a.rec + tileid) + 2, v0, v1);
                off = h0.x;
                nnz = h0.z;
                useful = rec_useful(h1, hit, (int)nnz);
                ++n_hit;
                n_hcol += __popc(hit);
            }
            int incl = useful;
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                const int v = __shfl_up_sync(0xffffffffu, incl, o);
                if (lane >= o) incl += v;
            }
            const int total = __shfl_sync(0xffffffffu, incl, 31);
            for (int q0 = 0; q0 < total; q0 += 32) {
                const int qv = q0 + lane;
                int lo = 0;
#pragma unroll
                for (int step = 16; step >= 1; step >>= 1) {
                    const int v = __shfl_sync(0xffffffffu, incl, lo + step - 1);
                    if (v <= qv) lo += step;
                }
                lo = min(lo, 31);
                const int exs = __shfl_sync(0xffffffffu, incl - useful, lo);
                const unsigned offs = __shfl_sync(0xffffffffu, off, lo);
                const int nns = __shfl_sync(0xffffffffu, (int)nnz, lo);
                const unsigned hs = __shfl_sync(0xffffffffu, hit, lo);
                const int os = __shfl_sync(0xffffffffu, ord, lo);
                const long long Js = __shfl_sync(0xffffffffu, J, lo);
                uint4 bs, w0, w1;
                bs.x = __shfl_sync(0xffffffffu, h1.x, lo);
                bs.y = __shfl_sync(0xffffffffu, h1.y, lo);
                bs.z = __shfl_sync(0xffffffffu, h1.z, lo);
                bs.w = __shfl_sync(0xffffffffu, h1.w, lo);
                w0.x = __shfl_sync(0xffffffffu, v0.x, lo);
                w0.y = __shfl_sync(0xffffffffu, v0.y, lo);
                w0.z = __shfl_sync(0xffffffffu, v0.z, lo);
                w0.w = __shfl_sync(0xffffffffu, v0.w, lo);
                w1.x = __shfl_sync(0xffffffffu, v1.x, lo);
                w1.y = __shfl_sync(0xffffffffu, v1.y, lo);
                w1.z = __shfl_sync(0xffffffffu, v1.z, lo);
                w1.w = __shfl_sync(0xffffffffu, v1.w, lo);
                if (qv < total) {
                    int pp, c, rr;
                    rec_position(bs, hs, nns, qv - exs, pp, c, rr);
                    if (rr < 0) rr = __ldg(&a.idx[offs + pp]) & (NT - 1);
                    double av = 1.0;
                    if (a.val) {
                        constexpr int INL = 32 / (int)sizeof(AV);
                        if (nns <= INL) {
                            if constexpr (sizeof(AV) == 8) {
                                const uint4 &vq = pp < 2 ? w0 : w1;
                                av = (pp & 1) ? __hiloint2double((int)vq.w, (int)vq.z)
                                              : __hiloint2double((int)vq.y, (int)vq.x);
                            } else {
                                const uint4 &vq = pp < 4 ? w0 : w1;
                                const int q4 = pp & 3;
                                av = (double)__uint_as_float(q4 == 0 ? vq.x : q4 == 1 ? vq.y : q4 == 2 ? vq.z : vq.w);
                            }
                        } else {
                            av = (double)__ldg(&((const AV *)a.val)[offs + pp]);
                            ++n_ind;
                        }
                    }
                    const double xv = __ldcg(&a.xd[Js * NT + c]);
                    ring_add<AV, SR>(ys + os * 16, yt + os, rr, av, xv);
                    ++n_mac;
                }
            }
            // next round's x-segment bits; its hit tiles' records are prefetched into
            // L2 while this round is flushed
            const unsigned xsn = In >= 0 ? xseg(a.xbits, Jn) : 0u;
            if (In >= 0 && (mkn & xsn)) asm volatile("prefetch.global.L2 [%0];" ::"l"(a.rec + idn));
            t += 32;
            __syncwarp();
            // row tiles before the first row tile of the next round are complete
            // (at the end of the range: all of them); the warp owns them, so each is
            // one coalesced read-modify-write of its 16 rows of acc
            const int nord = __popc(heads);
            const long long Inext = t < t1 ? (long long)__shfl_sync(0xffffffffu, In, 0) : -1;
            const int nfl = (t < t1 && rtI[nord - 1] == Inext) ? nord - 1 : nord;
            // rows the side merge (phase B) already touched: this half-word of the
            // touched bitmap (the other half belongs to the neighbouring row tile)
            unsigned sideb = 0;
            if (lane < nfl) {
                const long long Il = rtI[lane];
                sideb = (__ldcg(&a.rowbits[(Il * NT) >> 5]) >> ((Il & 1) * 16)) & 0xffffu;
            }
            for (int o = 0; o < nfl; o += 2) {
                const int so = o + (lane >> 4), r = lane & 15;
                const bool inr = so < nfl;
                const unsigned sb_o = __shfl_sync(0xffffffffu, sideb, min(so, 31));
                const long long Iq = inr ? rtI[so] : 0;
                const bool mine = inr && ((yt[so] >> r) & 1u);
                const long long row = Iq * NT + r;
                if (mine) {
                    const double v = ys[so * 16 + r];
                    if ((sb_o >> r) & 1u) {
                        const double old = a.acc[row];
                        if constexpr (SR == TSMV_PLUS_TIMES) {
                            a.acc[row] = old + v;
                        } else if constexpr (SR == TSMV_MIN_SECOND) {
                            a.acc[row] = __longlong_as_double(max(__double_as_longlong(old), __double_as_longlong(v)));
                        }
                    } else {
                        a.acc[row] = SR == TSMV_OR_AND ? __longlong_as_double(0ll) : v;
                        touch_row(a, s_pcnt, row);
                    }
                }
                if (inr) ys[so * 16 + r] = __longlong_as_double((long long)EMPTY);
                __syncwarp();
                if (inr && r == 0) yt[so] = 0u;
                __syncwarp();
            }
            if (nfl < nord) {
                // the last row tile continues in the next round: move it to slot 0
                const int sl = nord - 1;
                if (lane < 16 && sl > 0) {
                    ys[lane] = ys[sl * 16 + lane];
                    ys[sl * 16 + lane] = __longlong_as_double((long long)EMPTY);
                }
                __syncwarp();
                if (lane == 0 && sl > 0) {
                    yt[0] = yt[sl];
                    yt[sl] = 0u;
                    rtI[0] = rtI[sl];
                }
                __syncwarp();
            }
            I = In;
            J = Jn;
            mk = mkn;
            tileid = idn;
            xsg = xsn;
        }
    }
    // CTA statistics and the piece counts of rows this CTA touched first
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        n_hit += __shfl_xor_sync(0xffffffffu, n_hit, o);
        n_hcol += __shfl_xor_sync(0xffffffffu, n_hcol, o);
        n_mac += __shfl_xor_sync(0xffffffffu, n_mac, o);
        n_ind += __shfl_xor_sync(0xffffffffu, n_ind, o);
        n_seg += __shfl_xor_sync(0xffffffffu, n_seg, o);
    }
    if (lane == 0) {
        s_acct[wid][0] = n_hit;
        s_acct[wid][1] = n_hcol;
        s_acct[wid][2] = n_mac;
        s_acct[wid][3] = n_ind;
    }
    // per-warp x-side totals (lane values) into the per-CTA partials
    long long q4[4] = {n_seg, n_tiles, n_sent, n_side};
#pragma unroll
    for (int i = 2; i < 4; ++i)
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) q4[i] += __shfl_xor_sync(0xffffffffu, q4[i], o);
    __syncthreads();
    if (tid < 4) {
        long long sum = 0;
        for (int w = 0; w < RNW; ++w) sum += s_acct[w][tid];
        a.acct[b * 4 + tid] = sum;
    }
    __syncthreads();  // the sums above have read s_acct (compute-sanitizer racecheck, r2)
    if (lane == 0) {
        s_acct[wid][0] = q4[0];
        s_acct[wid][1] = q4[1];
        s_acct[wid][2] = q4[2];
        s_acct[wid][3] = q4[3];
    }
    __syncthreads();
    if (tid < 4) {
        long long sum = 0;
        for (int w = 0; w < RNW; ++w) sum += s_acct[w][tid];
        a.partials[b * 8 + tid] = sum;
    }
    if (!err)
        for (int q = tid; q < a.n_pieces; q += RT)
            if (s_pcnt[q]) atomicAdd(&a.pc[q], s_pcnt[q]);
    grid_sync_f(&a.cnt->bar, target, nullptr);
    const bool err2 = err;

    // ---------------------------------------------------------------- phase C (a6)
    // clear the x bitmap (every CTA has finished phase B), then compact y
    for (long long e = (long long)b * RT + tid; e < a.k; e += (long long)G * RT) {
        const long long j = a.x_idx[e];
        if (j >= 0 && j < a.n) a.xbits[j >> 5] = 0u;
    }
    long long yt = 0;
    {
        EmitArgs ea;
        ea.rowbits = a.rowbits;
        ea.acc = a.acc;
        ea.y_idx = a.y_idx;
        ea.y_val = a.y_val;
        ea.y_cap = a.y_cap;
        ea.row_begin = a.row_begin;
        ea.W = a.W;
        ea.pc = a.pc;
        ea.ps_log = a.ps_log;
        ea.n_pieces = a.n_pieces;
        ea.hy_idx = nullptr;  // host y by the copy kernel
        ea.hy_val = nullptr;
        // the ring accumulators are free now: they hold the dense-word lists
        long long *s_dw = reinterpret_cast<long long *>(s_dyn);
        long long *s_dpos = s_dw + RT;
        unsigned *s_dbits = reinterpret_cast<unsigned *>(s_dpos + RT);
        yt = emit_pieces<SR, XV, RT, RKP, RMAXG, RSPW, RBATCH>(ea, s_scan, s_pbase, s_ex0, s_tot, s_nd, s_dw,
                                                               s_dpos, s_dbits);
    }
    if (b == 0 && tid == 0) {
        a.cnt->y_nnz = yt;
        a.hm->y_nnz = yt;
        a.hm->err = err2 ? 1 : 0;
        if (a.ynnz_dev) *a.ynnz_dev = err2 ? -1 : yt;
        a.cnt->err = 0;
    }
}

template <class AV, class XV> void *pick_sr_rows(int sr) {
    if (sr == TSMV_PLUS_TIMES) return (void *)k_spmspv_rows<AV, XV, TSMV_PLUS_TIMES>;
    if (sr == TSMV_OR_AND) return (void *)k_spmspv_rows<AV, XV, TSMV_OR_AND>;
    return (void *)k_spmspv_rows<AV, XV, TSMV_MIN_SECOND>;
}
void *pick_rows(bool f32, int sr) { return f32 ? pick_sr_rows<float, float>(sr) : pick_sr_rows<double, double>(sr); }

constexpr size_t ROWS_DYN = (size_t)RNW * RING * 16 * 8 + (size_t)RNW * RING * 4 + (size_t)RMAXG * RKP * 4;
static_assert(ROWS_DYN <= 200 * 1024, "row kernel shared memory");
static_assert(ROWS_DYN >= (size_t)RT * 20, "phase C dense-word lists alias the ring accumulators");

void rows_set_smem() {
    static bool done = false;
    if (done) return;
    for (int f32 = 0; f32 < 2; ++f32)
        for (int sr = 0; sr < 3; ++sr)
            TSMV_CUDA(cudaFuncSetAttribute(pick_rows(f32, sr), cudaFuncAttributeMaxDynamicSharedMemorySize,
                                           (int)ROWS_DYN));
    done = true;
}

__global__ void k_rt_keys(const int32_t *__restrict__ trow, const int32_t *__restrict__ tgrp, int64_t T, int64_t nTC,
                          unsigned long long *__restrict__ keys, int32_t *__restrict__ ids) {
    for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < T; t += (int64_t)gridDim.x * blockDim.x) {
        keys[t] = (unsigned long long)trow[t] * (unsigned long long)nTC + (unsigned long long)tgrp[t];
        ids[t] = (int32_t)t;
    }
}
__global__ void k_rt_fill(const unsigned long long *__restrict__ keys, const int32_t *__restrict__ ids, int64_t T,
                          int64_t nTC, const uint16_t *__restrict__ mask, int32_t *__restrict__ rrow,
                          int32_t *__restrict__ rJ, uint16_t *__restrict__ rmask) {
    for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < T; t += (int64_t)gridDim.x * blockDim.x) {
        rrow[t] = (int32_t)(keys[t] / (unsigned long long)nTC);
        rJ[t] = (int32_t)(keys[t] % (unsigned long long)nTC);
        rmask[t] = mask[ids[t]];
    }
}

}  // namespace

// Row-major order of the dense tiles of P (tile row, then tile column) and the
// per-warp ranges of the row-driven kernel: equal tile counts per warp, cut at
// row-tile boundaries so that every row tile is summed by one warp.
void build_row_tiles(tsmv_ctx *c, cudaStream_t st) {
    TileSet &S = c->P;
    if (c->nt != 16 || !S.rec.p || S.T >= (1ll << 31)) return;
    const int64_t T = S.T;
    c->rows_G = std::min(c->sm_count, RMAXG);
    const long long nwarps = (long long)c->rows_G * RNW;
    c->rt_row.alloc(std::max<int64_t>(T, 1) * 4);
    c->rt_J.alloc(std::max<int64_t>(T, 1) * 4);
    c->rt_id.alloc(std::max<int64_t>(T, 1) * 4);
    c->rt_mask.alloc(std::max<int64_t>(T, 1) * 2);
    c->rt_wstart.alloc((nwarps + 1) * 8);
    std::vector<long long> ws(nwarps + 1, T);
    if (T > 0) {
        DevBuf kin, kout, idin, tmp;
        kin.alloc(T * 8);
        kout.alloc(T * 8);
        idin.alloc(T * 4);
        const int grid = (int)std::min<int64_t>((T + 255) / 256, 148 * 16);
        k_rt_keys<<<grid, 256, 0, st>>>(S.trow.as<int32_t>(), S.tgrp.as<int32_t>(), T, S.nTC,
                                         kin.as<unsigned long long>(), idin.as<int32_t>());
        TSMV_CUDA(cudaGetLastError());
        size_t tb = 0;
        TSMV_CUDA(cub::DeviceRadixSort::SortPairs(nullptr, tb, kin.as<unsigned long long>(),
                                                  kout.as<unsigned long long>(), idin.as<int32_t>(),
                                                  c->rt_id.as<int32_t>(), (int)T, 0, 64, st));
        tmp.alloc(tb);
        TSMV_CUDA(cub::DeviceRadixSort::SortPairs(tmp.p, tb, kin.as<unsigned long long>(),
                                                  kout.as<unsigned long long>(), idin.as<int32_t>(),
                                                  c->rt_id.as<int32_t>(), (int)T, 0, 64, st));
        k_rt_fill<<<grid, 256, 0, st>>>(kout.as<unsigned long long>(), c->rt_id.as<int32_t>(), T, S.nTC,
                                         S.mask.as<uint16_t>(), c->rt_row.as<int32_t>(), c->rt_J.as<int32_t>(),
                                         c->rt_mask.as<uint16_t>());
        TSMV_CUDA(cudaGetLastError());
        // warp ranges: equal tile counts, moved forward to the next row-tile start
        std::vector<int32_t> rows(T);
        TSMV_CUDA(cudaMemcpyAsync(rows.data(), c->rt_row.p, T * 4, cudaMemcpyDeviceToHost, st));
        TSMV_CUDA(cudaStreamSynchronize(st));
        ws[0] = 0;
        for (long long w = 1; w < nwarps; ++w) {
            long long t = std::max<long long>(ws[w - 1], (T * w) / nwarps);
            while (t < T && t > 0 && rows[t] == rows[t - 1]) ++t;
            ws[w] = t;
        }
        ws[nwarps] = T;
    }
    TSMV_CUDA(cudaMemcpyAsync(c->rt_wstart.p, ws.data(), (nwarps + 1) * 8, cudaMemcpyHostToDevice, st));
    TSMV_CUDA(cudaStreamSynchronize(st));
    const int64_t nw = (c->n + 31) / 32 + 1;
    c->xbits.alloc(nw * 4);
    TSMV_CUDA(cudaMemsetAsync(c->xbits.p, 0, c->xbits.bytes, st));
    c->use_rows = true;
}

// Density switch (measured on B200: profiles/r02_rows_vs_flat.txt).
// The row-driven kernel reads every dense tile (its cost ~ tiles per warp), the
// column-driven one only the tile columns of x's segments plus one atomic per
// useful nonzero.  Row-driven when the matrix keeps almost all nonzeros in tiles
// (side matrix <= 10 %), the tiles are not dense blocks (<= 32 nonzeros on
// average: dense band tiles turn into long multiply rounds) and either x's
// density is at least tsmv_options.row_driven_density (default 0.05: 3D stencil
// 1.19 vs 1.33 ms at 10 %, 2D 26 vs 38 us) or the whole tile list is one round
// per warp (small matrices: 2D 64x64 at 1 %, 25 vs 32 us).  0 = never;
// TSMV_SPMSPV_KERNEL=rows|flat forces one (tests, ablation).
bool use_rows_kernel(const tsmv_ctx *c, long long k) {
    if (!c->use_rows) return false;
    if (const char *f = getenv("TSMV_SPMSPV_KERNEL")) return f[0] == 'r';
    const double d = c->opt.row_driven_density;
    if (d <= 0) return false;
    const TileSet &S = c->P;
    const long long nnz = S.dense_nnz + S.side_nnz;
    if (S.T == 0 || (double)S.side_nnz > 0.1 * (double)nnz || S.dense_nnz > 32 * S.T) return false;
    const bool small = S.T <= 32ll * c->rows_G * RNW;
    return small || (double)k >= d * (double)c->n;
}

void enqueue_spmspv_rows(tsmv_ctx *c, int sr, long long k, const int32_t *xi, const void *xv, long long ycap,
                         int32_t *yi, void *yv, long long *ynnz_dev, cudaStream_t st) {
    const bool f32 = c->dtype == TSMV_F32;
    RowArgs a;
    a.x_idx = xi;
    a.x_val = xv;
    a.k = k;
    a.n = c->n;
    a.m = c->m;
    a.W = (c->m + 31) / 32;
    a.row_begin = c->row_begin;
    a.rrow = c->rt_row.as<int32_t>();
    a.rJ = c->rt_J.as<int32_t>();
    a.rid = c->rt_id.as<int32_t>();
    a.rmask = c->rt_mask.as<uint16_t>();
    a.wstart = c->rt_wstart.as<long long>();
    a.rec = c->P.rec.as<TileRec64>();
    a.idx = c->P.idx.as<uint8_t>();
    a.val = c->P.has_vals ? c->P.val.p : nullptr;
    a.sptr = c->P.sptr.as<long long>();
    a.srow = c->P.srow.as<int>();
    a.sval = c->P.has_vals ? c->P.sval.p : nullptr;
    a.hot_list = c->P.hot_list;
    a.n_hot = c->P.hot_list ? c->n_hot : 0;
    a.xd = c->xdense.as<double>();
    a.xbits = c->xbits.as<uint32_t>();
    a.acc = c->acc.as<double>();
    a.rowbits = c->rowbits_p;
    {
        const int G = c->rows_G;
        const long long per = (a.W + (long long)G * RKP - 1) / ((long long)G * RKP);
        int lg = 5;
        while ((1ll << lg) < per) ++lg;
        a.ps_log = lg;
        a.n_pieces = (int)((a.W + (1ll << lg) - 1) >> lg);
        unsigned *pc = c->FL.pcnt.as<unsigned>();
        const int cur = (int)(c->flat_calls & 1);
        a.pc = pc + (size_t)cur * RMAXG * RKP;
        a.pc_next = pc + (size_t)(1 - cur) * RMAXG * RKP;
        c->flat_calls++;
    }
    a.y_idx = yi;
    a.y_val = (sr == TSMV_OR_AND) ? nullptr : yv;
    a.y_cap = ycap;
    a.ynnz_dev = ynnz_dev;
    a.partials = c->partials.as<long long>();
    a.acct = c->acct.as<long long>();
    a.cnt = c->counters.as<Counters>();
    a.hm = c->hcnt_dev;
    a.bar_base = c->bar_base;
    rows_set_smem();
    void *args[] = {&a};
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(c->rows_G);
    cfg.blockDim = dim3(RT);
    cfg.dynamicSmemBytes = ROWS_DYN;
    cfg.stream = st;
    cudaLaunchAttribute at[2];
    at[0].id = cudaLaunchAttributeCooperative;
    at[0].val.cooperative = 1;
    cfg.numAttrs = 1;
    if (c->persist_bytes) {
        at[1].id = cudaLaunchAttributeAccessPolicyWindow;
        at[1].val.accessPolicyWindow.base_ptr = c->acc.p;
        at[1].val.accessPolicyWindow.num_bytes = c->persist_bytes;
        at[1].val.accessPolicyWindow.hitRatio = c->persist_ratio;
        at[1].val.accessPolicyWindow.hitProp = cudaAccessPropertyPersisting;
        at[1].val.accessPolicyWindow.missProp = cudaAccessPropertyStreaming;
        cfg.numAttrs = 2;
    }
    cfg.attrs = at;
    TSMV_CUDA(cudaLaunchKernelExC(&cfg, pick_rows(f32, sr), args));
    c->bar_base += 3ull * (unsigned long long)c->rows_G;
    c->last_blocks = c->rows_G;
}

}  // namespace tsmv
