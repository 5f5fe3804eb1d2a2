// spmspv_common.cuh -- device pieces shared by the column-driven (flat,
// spmspv_flat.cu) and the row-driven (Alg 4, spmspv_rows.cu) TileSpMSpV kernels:
// the accumulator encoding with exact first-touch detection, tile-record
// helpers, the grid barrier, and phase C (y compaction from the touched-row
// bitmap).
#pragma once
#include "device.cuh"

namespace tsmv {
namespace {

// Accumulator encoding (all semirings): an untouched row holds EMPTY = the bits
// of -0.0, which is the identity of both updates used here: -0.0 + v == v (plus-
// times, fp64), and LLONG_MIN is the identity of a signed max, to which the
// min-second keys are mapped (k' = ~ord_key(x) ^ 2^63 keeps the order).  The old
// value returned by the atomic tells whether this contribution is the first to
// its row; only that one sets the row's touched bit and counts the row in its
// bitmap piece (one RED.OR + one RED.ADD per output row instead of one per
// contribution).  The detection is exact: a zero product is added as +0.0, so
// after its first contribution a row never holds -0.0 again (x + (-x) = +0.0
// under round-to-nearest); Boolean rows are claimed with an exchange; a min key
// never equals EMPTY (it would need an all-ones order key, i.e. a NaN x).
constexpr unsigned long long EMPTY = 0x8000000000000000ull;

__device__ __forceinline__ double prod_nz(double a, double x) {
    const double v = a * x;
    return v == 0.0 ? 0.0 : v;  // -0.0 -> +0.0
}
template <int SR>
__device__ __forceinline__ bool acc_first(double *acc, long long row, double a, double x) {
    if constexpr (SR == TSMV_PLUS_TIMES) {
        return (unsigned long long)__double_as_longlong(atomicAdd(&acc[row], prod_nz(a, x))) == EMPTY;
    } else if constexpr (SR == TSMV_MIN_SECOND) {
        const long long k = (long long)(~ord_key(x) ^ EMPTY);
        return (unsigned long long)atomicMax((long long *)&acc[row], k) == EMPTY;
    } else {
        return atomicExch((unsigned long long *)&acc[row], 0ull) == EMPTY;
    }
}
template <int SR>
__device__ __forceinline__ void acc_shared(double *s, int slot, double a, double x) {
    if constexpr (SR == TSMV_PLUS_TIMES) atomicAdd(&s[slot], prod_nz(a, x));
    else if constexpr (SR == TSMV_MIN_SECOND) atomicMax((long long *)&s[slot], (long long)(~ord_key(x) ^ EMPTY));
}

// 32-byte read-only load (one LDG.E.ENL2.256 request instead of two 16-byte ones)
__device__ __forceinline__ void ld32_nc(const void *p, uint4 &lo, uint4 &hi) {
    asm volatile("ld.global.nc.v8.u32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
                 : "=r"(lo.x), "=r"(lo.y), "=r"(lo.z), "=r"(lo.w), "=r"(hi.x), "=r"(hi.y), "=r"(hi.z), "=r"(hi.w)
                 : "l"(p));
}

__device__ __forceinline__ int byte_of(const uint4 &w, int i) {
    const unsigned x = i < 8 ? (i < 4 ? w.x : w.y) : (i < 12 ? w.z : w.w);
    return (int)((x >> ((i & 3) * 8)) & 0xffu);
}
// column start c of a tile with cstart bytes in w (c == 16 -> nnz)
__device__ __forceinline__ int cs_of(const uint4 &w, int c, int nnz) { return c >= 16 ? nnz : byte_of(w, c); }

// Inline index bytes (nnz <= 16) are (c << 4) | r in column-major order, padding
// bytes are 0xff.  cw = their column nibbles, four per word, so that the count of
// bytes in / before a column is a SIMD byte compare + popc (no per-byte loop).
__device__ __forceinline__ void col_nibbles(const uint4 &b, unsigned (&cw)[4]) {
    cw[0] = (b.x >> 4) & 0x0f0f0f0fu;
    cw[1] = (b.y >> 4) & 0x0f0f0f0fu;
    cw[2] = (b.z >> 4) & 0x0f0f0f0fu;
    cw[3] = (b.w >> 4) & 0x0f0f0f0fu;
}
// bytes i < nnz with column c
__device__ __forceinline__ int count_col_eq(const unsigned (&cw)[4], int c, int nnz) {
    const unsigned rep = 0x01010101u * (unsigned)c;
    int s = 0;
#pragma unroll
    for (int i = 0; i < 4; ++i) {
        const int v = nnz - 4 * i;
        const unsigned vm = v >= 4 ? 0xffffffffu : (v <= 0 ? 0u : (0xffffffffu >> (32 - 8 * v)));
        s += __popc(__vcmpeq4(cw[i], rep) & vm);
    }
    return s >> 3;
}
// bytes with column < c (padding has column 15 and is never counted for c <= 15)
__device__ __forceinline__ int count_col_lt(const unsigned (&cw)[4], int c) {
    const unsigned rep = 0x01010101u * (unsigned)c;
    int s = 0;
#pragma unroll
    for (int i = 0; i < 4; ++i) s += __popc(__vcmpltu4(cw[i], rep));
    return s >> 3;
}

// Useful nonzeros of a hit tile (nonzeros in the columns of `hit`).
__device__ __forceinline__ int rec_useful(const uint4 &b, unsigned hit, int nnz) {
    int s = 0;
    if (nnz <= 16) {
        unsigned cw[4];
        col_nibbles(b, cw);
        while (hit) {
            const int c = __ffs(hit) - 1;
            hit &= hit - 1;
            s += count_col_eq(cw, c, nnz);
        }
    } else {
        while (hit) {
            const int c = __ffs(hit) - 1;
            hit &= hit - 1;
            s += cs_of(b, c + 1, nnz) - cs_of(b, c, nnz);
        }
    }
    return s;
}

// Position p (in the tile's nonzeros) and column c of the k-th useful nonzero.
// For nnz <= 16 also its row r (from the inline index byte); else r = -1.
__device__ __forceinline__ void rec_position(const uint4 &b, unsigned hit, int nnz, int k, int &p, int &c, int &r) {
    p = 0;
    c = 0;
    r = -1;
    if (nnz <= 16) {
        unsigned cw[4];
        col_nibbles(b, cw);
        while (hit) {
            c = __ffs(hit) - 1;
            hit &= hit - 1;
            const int len = count_col_eq(cw, c, nnz);
            if (k < len) {
                p = count_col_lt(cw, c) + k;
                r = byte_of(b, p) & 15;
                return;
            }
            k -= len;
        }
        return;
    }
    while (hit) {
        c = __ffs(hit) - 1;
        hit &= hit - 1;
        const int p0 = cs_of(b, c, nnz), len = cs_of(b, c + 1, nnz) - p0;
        if (k < len) {
            p = p0 + k;
            return;
        }
        k -= len;
    }
}

// tr (CTA-private, may be null): [0] = arrival of the whole CTA, [1] = release seen
__device__ __forceinline__ void grid_sync_f(unsigned long long *bar, unsigned long long &target,
                                            unsigned long long *tr) {
    __syncthreads();
    target += gridDim.x;
    if (threadIdx.x == 0) {
        if (tr) tr[0] = globaltimer_ns();
        __threadfence();
        atomicAdd(bar, 1ull);
        while (ld_acquire_u64(bar) < target) {
        }
        __threadfence();
        if (tr) tr[1] = globaltimer_ns();
    }
    __syncthreads();
}


// Phase C (a6): y compaction.  The touched bitmap is cut into pieces of
// PS = 2^ps_log words (at most G*KP of them); CTA b owns pieces b, b + G, ..., so
// a dense stretch of y (power-law rows) is spread over KP CTAs.  The rows of
// every piece were counted at their first touch, so each CTA scans the piece
// counts and emits its pieces at their global offsets.  A round covers PSR
// words of each of the CTA's pieces (thread tid: piece tid / PSR), so one block
// scan per round serves all pieces.  Sparse words (<= SPW set rows) are emitted
// by their own thread, dense ones by whole warps (coalesced acc loads, y stores).
// acc and the bitmap are cleared on read.  Returns y_nnz (all threads).
struct EmitArgs {
    uint32_t *rowbits;
    double *acc;
    int32_t *y_idx;
    void *y_val;
    long long y_cap, row_begin, W;
    const unsigned *pc;
    int ps_log, n_pieces;
    int32_t *hy_idx;  // mapped pinned host y (or null): each CTA copies its pieces' rows there
    void *hy_val;     // once they are emitted (coalesced, overlapping the other CTAs' work)
};
template <int SR, class XV, int FT, int KP, int MAXG, int SPW, int BATCH>
__device__ long long emit_pieces(const EmitArgs &a, long long (*s_scan)[FT / 32], long long *s_pbase,
                                 long long *s_ex0, long long *s_tot, int &s_nd, long long *s_dw, long long *s_dpos,
                                 unsigned *s_dbits) {
    constexpr int NWF = FT / 32;
    const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
    const int G = gridDim.x, b = blockIdx.x;
    constexpr int PSR = FT / KP;
    const long long PS = 1ll << a.ps_log;
    const int kp = tid / PSR, tp = tid % PSR;
    const long long pw0 = ((long long)b + (long long)kp * G) * PS;
    const long long pw1 = min(a.W, pw0 + PS);
    // the first round's bitmap words do not depend on the piece counts: loaded
    // before the counts' scan, so the two round trips overlap
    const unsigned bits_r0 = pw0 + tp < pw1 ? __ldcg(&a.rowbits[pw0 + tp]) : 0u;
    {
        // exclusive prefix of all piece counts (every CTA, in shared memory)
        const int NP = a.n_pieces;
        constexpr int PPT = (MAXG * KP + FT - 1) / FT;
        long long v[PPT], run = 0;
#pragma unroll
        for (int i = 0; i < PPT; ++i) {
            const int q = tid * PPT + i;
            v[i] = q < NP ? (long long)__ldcg(&a.pc[q]) : 0;
            run += v[i];
        }
        long long ex, tt;
        block_scan<1, FT>(&run, &ex, &tt, s_scan);
        if (tid < KP) s_pbase[tid] = 0;
        __syncthreads();
#pragma unroll
        for (int i = 0; i < PPT; ++i) {
            const int q = tid * PPT + i;
            if (q < NP && (q % G) == b) s_pbase[q / G] = ex;
            ex += v[i];
        }
        if (tid == 0) s_tot[0] = tt;
    }
    __syncthreads();
    __shared__ long long s_pst[KP];  // first output position of each of the CTA's pieces
    if (tid < KP) s_pst[tid] = s_pbase[tid];
    const long long ycap = a.y_cap;
    const int nround = (int)((PS + PSR - 1) / PSR);
    if (tid == 0) s_nd = 0;
    for (int rd = 0; rd < nround; ++rd) {
        const long long w = pw0 + (long long)rd * PSR + tp;
        const unsigned bits = rd == 0 ? bits_r0 : (w < pw1 ? __ldcg(&a.rowbits[w]) : 0u);
        long long c = __popc(bits), exw, rtot;
        block_scan<1, FT>(&c, &exw, &rtot, s_scan);
        if (tp == 0) s_ex0[kp] = exw;
        __syncthreads();
        const long long seg0 = s_ex0[kp];
        const long long segsum = (kp + 1 < KP ? s_ex0[kp + 1] : rtot) - seg0;
        const long long pos0 = s_pbase[kp] + exw - seg0;
        __syncthreads();
        if (tp == 0) s_pbase[kp] += segsum;
        int it = 0;
        if (bits) a.rowbits[w] = 0u;
        // sparse words (<= SPW set rows) are emitted by their own thread, all in one
        // round of independent loads; dense words by the whole warp, BATCH words per
        // round, lane l handling row l (coalesced acc loads and y stores)
        const int pc = __popc(bits);
        if (pc > 0 && pc <= SPW) {
            unsigned bb = bits;
            int rr[SPW];
            double v[SPW];
#pragma unroll
            for (int kk = 0; kk < SPW; ++kk) {
                rr[kk] = bb ? __ffs(bb) - 1 : 0;
                bb &= bb - 1;
            }
#pragma unroll
            for (int kk = 0; kk < SPW; ++kk)
                if (kk < pc) v[kk] = __ldcg(&a.acc[w * 32 + rr[kk]]);
#pragma unroll
            for (int kk = 0; kk < SPW; ++kk) {
                if (kk < pc) {
                    const long long row = w * 32 + rr[kk];
                    const long long pos = pos0 + kk;
                    a.acc[row] = __longlong_as_double((long long)EMPTY);
                    if (pos < ycap) {
                        a.y_idx[pos] = (int32_t)(row + a.row_begin);
                        if (a.y_val) {
                            double x = v[kk];
                            if constexpr (SR == TSMV_MIN_SECOND)
                                x = ord_val(~((unsigned long long)__double_as_longlong(x) ^ EMPTY));
                            ((XV *)a.y_val)[pos] = (XV)x;
                        }
                    }
                }
            }
        }
        // dense words (> SPW set rows) go to a CTA list and are emitted by all warps
        // of the CTA, BATCH words per warp and round, lane l handling row l
        // (coalesced acc loads and y stores): a dense stretch of y owned by a few
        // threads of one piece is spread over the whole CTA
        if (pc > SPW) {
            const int q = atomicAdd(&s_nd, 1);
            s_dw[q] = w;
            s_dpos[q] = pos0;
            s_dbits[q] = bits;
        }
        __syncthreads();
        const int nd = s_nd;
        const unsigned lt = (1u << lane) - 1u;
        for (int q0 = wid * BATCH; q0 < nd; q0 += NWF * BATCH) {
            long long wq[BATCH];
            unsigned bq[BATCH];
            double v[BATCH];
            bool mine[BATCH];
#pragma unroll
            for (int kk = 0; kk < BATCH; ++kk) {
                const int q = q0 + kk;
                wq[kk] = q < nd ? s_dw[q] : 0;
                bq[kk] = q < nd ? s_dbits[q] : 0u;
                mine[kk] = (bq[kk] >> lane) & 1u;
                if (mine[kk]) v[kk] = __ldcg(&a.acc[wq[kk] * 32 + lane]);
            }
#pragma unroll
            for (int kk = 0; kk < BATCH; ++kk) {
                if (mine[kk]) {
                    const long long row = wq[kk] * 32 + lane;
                    const long long pos = s_dpos[q0 + kk] + __popc(bq[kk] & lt);
                    a.acc[row] = __longlong_as_double((long long)EMPTY);
                    if (pos < ycap) {
                        a.y_idx[pos] = (int32_t)(row + a.row_begin);
                        if (a.y_val) {
                            double x = v[kk];
                            if constexpr (SR == TSMV_MIN_SECOND)
                                x = ord_val(~((unsigned long long)__double_as_longlong(x) ^ EMPTY));
                            ((XV *)a.y_val)[pos] = (XV)x;
                        }
                    }
                }
            }
        }
        __syncthreads();
        if (tid == 0) s_nd = 0;
    }
    __syncthreads();
    if (a.hy_idx || a.hy_val) {
        // the CTA's pieces are complete: their rows [s_pst, s_pbase) of y go to the
        // host buffers now (consecutive threads, consecutive addresses), while other
        // CTAs still emit (no copy kernel behind the call)
        const long long nb = (long long)b;
        for (int q = 0; q < KP; ++q) {
            if (nb + (long long)q * G >= a.n_pieces) break;
            const long long lo = s_pst[q], hi = min(s_pbase[q], ycap);
            for (long long i = lo + tid; i < hi; i += FT) {
                if (a.hy_idx) a.hy_idx[i] = __ldcg(&a.y_idx[i]);
                if (a.hy_val && a.y_val) ((XV *)a.hy_val)[i] = __ldcg(&((const XV *)a.y_val)[i]);
            }
        }
    }
    return s_tot[0];
}

}  // namespace
}  // namespace tsmv
