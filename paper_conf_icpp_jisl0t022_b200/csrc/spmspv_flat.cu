// spmspv_flat.cu -- TileSpMSpV y = A x, "flat" cooperative kernel for nt = 16
// (Sec 3.3, tiled vector Sec 3.2.2
// P:533-573, semirings P:1373-1379).
//
// Why a second kernel: B200 measurements (profiles/r01_summary.md, round-1
// session 2) put the cost of this irregular path in (i) dependent HBM hops and
// (ii) the random-sector rate (~40 G sectors/s cold, only at high memory-level
// parallelism).  The first fused kernel ran 16 warps/SM and let one warp walk a
// 128-item chunk of power-law hub tiles in ~11 dependent rounds.  This kernel:
//   * 32 warps per SM (1024-thread CTAs, 64 registers), so twice the loads in flight;
//   * phase A reserves list slots with ONE 64-bit atomic per CTA on a packed
//     (count, work) counter instead of a grid-wide scan + barrier: slot order and
//     work order agree, which is all the chunk maps need (accumulation order is free);
//   * tile work in 32-item warp chunks: lane = tile item, mask test, then one
//     32-byte TileRec16 per hit (descriptor + the tile's 16 index bytes inline when
//     nnz <= 16, else its 16 column starts), and the useful nonzeros of the warp's
//     hit tiles are redistributed over the lanes with shuffles (no shared memory);
//   * side work (very sparse tiles, Alg 2 column merge) in 128-item chunks whose
//     list window (start, x_j) is staged in shared memory;
//   * chunks are dealt round-robin to warps (no work-queue atomics on one address);
//   * compaction with one thread per bitmap word (loads of its set rows batched).
// Phases: A | barrier | B (a3-a5) | barrier | C1 count | barrier | C2 write y.
#include "device.cuh"
#include <algorithm>
#include <cstdlib>

namespace tsmv {

namespace {

constexpr int FT = 1024;          // threads per CTA
constexpr int NWF = FT / 32;      // warps per CTA
constexpr int TL = 5;             // log2 tile items per warp chunk
constexpr int SL = 7;             // log2 side items per warp chunk
constexpr int US = (1 << SL) / 32;
constexpr int BATCH = 8;          // accumulator loads in flight per thread in C2
constexpr int FLAT_TRING = 4096;
constexpr unsigned long long T_CNT_SHIFT = 40, S_CNT_SHIFT = 37;
constexpr long long INF64 = 0x7fffffffffffffffLL;

struct FlatArgs {
    const int32_t *x_idx;
    const void *x_val;
    long long k, n, m, W, row_begin;
    const long long *tptr;
    const uint16_t *mask;
    const TileRec16 *rec;
    const uint8_t *idx;
    const void *val;
    const long long *sptr;
    const int *srow;
    const void *sval;
    FlatListsView L;
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
    unsigned long long *tring;
    long long tslot;
    const int32_t *hot_list;
    int n_hot;
    unsigned long long *trace;  // tsmv_set_trace: per CTA 8 globaltimer stamps (dev aid)
};

template <int SR>
__device__ __forceinline__ void acc_global(double *acc, long long row, double a, double x) {
    if constexpr (SR == TSMV_PLUS_TIMES) atomicAdd(&acc[row], a * x);
    else if constexpr (SR == TSMV_MIN_SECOND) atomicMax((unsigned long long *)&acc[row], ~ord_key(x));
}
template <int SR>
__device__ __forceinline__ void acc_shared(double *s, int slot, double a, double x) {
    if constexpr (SR == TSMV_PLUS_TIMES) atomicAdd(&s[slot], a * x);
    else if constexpr (SR == TSMV_MIN_SECOND) atomicMax((unsigned long long *)&s[slot], ~ord_key(x));
}

// One contribution a*x to row code `rc` (>= 0: local row; < 0: ~hot slot).
template <int SR>
__device__ __forceinline__ void contribute(const FlatArgs &a, double *s_hacc, uint32_t *s_hbits, long long rc,
                                           double av, double xv) {
    if (rc < 0) {
        const int sl = (int)~rc;
        acc_shared<SR>(s_hacc, sl, av, xv);
        atomicOr(&s_hbits[sl >> 5], 1u << (sl & 31));
    } else {
        acc_global<SR>(a.acc, rc, av, xv);
        atomicOr(&a.rowbits[rc >> 5], 1u << (rc & 31));
    }
}

#ifdef TSMV_FLAT_STEPS
// development: stamp step k of the warp that processes tile chunk 0 once the value
// `dep` (produced by the step's loads) is available
#define FSTEP(k, dep)                                                                              \
    do {                                                                                           \
        if (a.trace && ch == 0 && lane == 0) {                                                     \
            if ((long long)(dep) == 0x5eed5eed5eedll) a.trace[2000] = 1;                          \
            a.trace[148 * 8 + (k)] = globaltimer_ns();                                             \
        }                                                                                          \
    } while (0)
#define CSTEP(k, dep)                                                                              \
    do {                                                                                           \
        if (a.trace && b == 1 && wid == 0 && lane == 0 && (k) < 16) {                              \
            if ((long long)(dep) == 0x5eed5eed5eedll) a.trace[2000] = 1;                          \
            a.trace[148 * 8 + 16 + (k)] = globaltimer_ns();                                        \
        }                                                                                          \
    } while (0)
#else
#define FSTEP(k, dep) ((void)0)
#define CSTEP(k, dep) ((void)0)
#endif

constexpr int HEAVY_CAP = 128;
// Chunk -> list-entry map for an entry owning work items [w0, w0 + w): short runs
// are written by the calling thread, long ones are queued for a warp.
template <int LOGC>
__device__ __forceinline__ void put_chunks(int *C, long long w0, long long w, int entry, int kind,
                                           long long (*heavy)[3], int *nheavy) {
    constexpr int CH = 1 << LOGC;
    const long long c0 = (w0 + CH - 1) >> LOGC, c1 = (w0 + w + CH - 1) >> LOGC;
    if (c1 - c0 > 4) {
        const int q = atomicAdd(nheavy, 1);
        if (q < HEAVY_CAP) {
            heavy[q][0] = c0;
            heavy[q][1] = c1;
            heavy[q][2] = ((long long)kind << 32) | (unsigned)entry;
            return;
        }
    }
    for (long long ch = c0; ch < c1; ++ch) C[ch] = entry;
}

__device__ __forceinline__ int byte_of(const uint4 &w, int i) {
    const unsigned x = i < 8 ? (i < 4 ? w.x : w.y) : (i < 12 ? w.z : w.w);
    return (int)((x >> ((i & 3) * 8)) & 0xffu);
}
// column start c of a tile with cstart bytes in w (c == 16 -> nnz)
__device__ __forceinline__ int cs_of(const uint4 &w, int c, int nnz) { return c >= 16 ? nnz : byte_of(w, c); }

// Useful nonzeros of a hit tile (nonzeros in the columns of `hit`).
__device__ __forceinline__ int rec_useful(const uint4 &b, unsigned hit, int nnz) {
    int s = 0;
    if (nnz <= 16) {
#pragma unroll
        for (int i = 0; i < 16; ++i)
            if (i < nnz) s += (hit >> (byte_of(b, i) >> 4)) & 1u;
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
#pragma unroll
        for (int i = 0; i < 16; ++i) {
            if (i < nnz) {
                const int v = byte_of(b, i);
                if ((hit >> (v >> 4)) & 1u) {
                    if (k == 0) {
                        p = i;
                        c = v >> 4;
                        r = v & 15;
                    }
                    --k;
                }
            }
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

template <class AV, class XV, int SR>
__global__ void __launch_bounds__(FT, 1) k_spmspv_flat(FlatArgs a) {
    constexpr int NT = 16, LOG = 4;
    constexpr int WN = (1 << SL) + 1;
    __shared__ long long s_scan[8][NWF];
    extern __shared__ __align__(16) unsigned char s_dyn[];
    double *s_hacc = reinterpret_cast<double *>(s_dyn);                           // [HOT_SLOTS]
    long long *s_win = reinterpret_cast<long long *>(s_dyn + HOT_SLOTS * 8);      // [NWF][WN]
    long long *s_winb = s_win + NWF * WN;                                         // [NWF][WN]
    double *s_winx = reinterpret_cast<double *>(s_winb + NWF * WN);               // [NWF][WN]
    uint32_t *s_hbits = reinterpret_cast<uint32_t *>(s_winx + NWF * WN);          // [HOT_SLOTS/32]
    __shared__ long long s_base[4], s_tot[4];
    __shared__ long long s_acct[NWF][3];
    __shared__ int s_err;
    __shared__ int s_nheavy;
    __shared__ long long s_heavy[HEAVY_CAP][3];  // chunk-map runs too long for one thread: c0, c1, list | kind
    const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
    const int G = gridDim.x, b = blockIdx.x;
    unsigned long long target = a.bar_base;
    const bool stamp = a.tring && b == 0 && tid == 0;
    unsigned long long *ts = a.tring ? a.tring + (a.tslot % FLAT_TRING) * 8 : nullptr;
    if (stamp) ts[0] = globaltimer_ns();
    unsigned long long *tr = a.trace ? a.trace + (long long)b * 8 : nullptr;
    if (tr && tid == 0) tr[0] = globaltimer_ns();
    const int n_slots = a.n_hot * NT;
    for (int i = tid; i < n_slots; i += FT) s_hacc[i] = 0.0;
    for (int i = tid; i < (n_slots + 31) / 32; i += FT) s_hbits[i] = 0u;
    if (tid == 0) s_nheavy = 0;

    // ------------------------------------------------------------ phase A (a2)
    // CTA b owns x entries [e0, e1); thread tid a contiguous run of them.
    const long long E = (a.k + G - 1) / G;
    const long long e0 = (long long)b * E, e1 = min(a.k, e0 + E);
    const long long per = (E + FT - 1) / FT;
    const long long te0 = min(e1, e0 + tid * per), te1 = min(e1, te0 + per);
    long long q[4] = {0, 0, 0, 0};  // tile entries, tile work, side entries, side work
    bool bad_any = false;
    for (long long e = te0; e < te1; ++e) {
        const long long j = a.x_idx[e];
        const long long prev = e > 0 ? (long long)a.x_idx[e - 1] : -1;
        const bool bad = j < 0 || j >= a.n || prev >= j;
        bad_any |= bad;
        if (bad) continue;
        const long long J = j >> LOG;
        if (e == 0 || (prev >> LOG) != J) {
            const long long wt = a.tptr[J + 1] - a.tptr[J];
            q[0] += wt > 0;
            q[1] += wt;
        }
        const long long ws = a.sptr[j + 1] - a.sptr[j];
        q[2] += ws > 0;
        q[3] += ws;
        a.L.xd[j] = a.x_val ? (double)((const XV *)a.x_val)[e] : 1.0;
    }
    if (bad_any) a.cnt->err = 1;
    long long ex[4], tot[4];
    block_scan<4, FT>(q, ex, tot, s_scan);
    if (tid == 0) {
        // reserve this CTA's slots and work ranges: one packed atomic per list
        const unsigned long long ot =
            atomicAdd(&a.cnt->resv_t, ((unsigned long long)tot[0] << T_CNT_SHIFT) | (unsigned long long)tot[1]);
        const unsigned long long os =
            atomicAdd(&a.cnt->resv_s, ((unsigned long long)tot[2] << S_CNT_SHIFT) | (unsigned long long)tot[3]);
        s_base[0] = (long long)(ot >> T_CNT_SHIFT);
        s_base[1] = (long long)(ot & ((1ull << T_CNT_SHIFT) - 1));
        s_base[2] = (long long)(os >> S_CNT_SHIFT);
        s_base[3] = (long long)(os & ((1ull << S_CNT_SHIFT) - 1));
#pragma unroll
        for (int i = 0; i < 4; ++i) a.partials[b * 8 + i] = tot[i];
    }
    __syncthreads();
    {
        long long oLt = s_base[0] + ex[0], oWt = s_base[1] + ex[1];
        long long oLs = s_base[2] + ex[2], oWs = s_base[3] + ex[3];
        for (long long e = te0; e < te1; ++e) {
            const long long j = a.x_idx[e];
            const long long prev = e > 0 ? (long long)a.x_idx[e - 1] : -1;
            if (j < 0 || j >= a.n || prev >= j) continue;
            const long long J = j >> LOG;
            if (e == 0 || (prev >> LOG) != J) {
                const long long tb = a.tptr[J], wt = a.tptr[J + 1] - tb;
                if (wt > 0) {
                    unsigned mk = 0;
                    for (long long e2 = e; e2 < a.k; ++e2) {
                        const long long j2 = a.x_idx[e2];
                        if ((j2 >> LOG) != J) break;
                        mk |= 1u << (j2 & (NT - 1));
                    }
                    a.L.t_beg[oLt] = tb;
                    a.L.t_wpre[oLt] = oWt;
                    a.L.t_xm[oLt] = mk;
                    a.L.t_J[oLt] = (int)J;
                    put_chunks<TL>(a.L.Ct, oWt, wt, (int)oLt, 0, s_heavy, &s_nheavy);
                    ++oLt;
                    oWt += wt;
                }
            }
            const long long sb = a.sptr[j], ws = a.sptr[j + 1] - sb;
            if (ws > 0) {
                a.L.s_beg[oLs] = sb;
                a.L.s_wpre[oLs] = oWs;
                a.L.s_x[oLs] = a.x_val ? (double)((const XV *)a.x_val)[e] : 1.0;
                put_chunks<SL>(a.L.Cs, oWs, ws, (int)oLs, 1, s_heavy, &s_nheavy);
                ++oLs;
                oWs += ws;
            }
        }
    }
    __syncthreads();
    {
        // long chunk-map runs (hub columns) written by a whole warp
        const int nh = min(s_nheavy, HEAVY_CAP);
        for (int h = wid; h < nh; h += NWF) {
            int *C = s_heavy[h][2] >> 32 ? a.L.Cs : a.L.Ct;
            const int entry = (int)(s_heavy[h][2] & 0xffffffffll);
            for (long long ch = s_heavy[h][0] + lane; ch < s_heavy[h][1]; ch += 32) C[ch] = entry;
        }
    }
    grid_sync_f(&a.cnt->bar, target, tr ? tr + 1 : nullptr);
    if (stamp) ts[1] = globaltimer_ns();
    if (tid == 0) {
        const unsigned long long rt = __ldcg(&a.cnt->resv_t), rs = __ldcg(&a.cnt->resv_s);
        s_tot[0] = (long long)(rt >> T_CNT_SHIFT);
        s_tot[1] = (long long)(rt & ((1ull << T_CNT_SHIFT) - 1));
        s_tot[2] = (long long)(rs >> S_CNT_SHIFT);
        s_tot[3] = (long long)(rs & ((1ull << S_CNT_SHIFT) - 1));
        s_err = __ldcg(&a.cnt->err);
    }
    __syncthreads();
    const bool err = s_err != 0;
    if (stamp) ts[2] = globaltimer_ns();

    // ------------------------------------------------------------ phase B (a3-a5)
    long long n_hit = 0, n_hcol = 0, n_mac = 0;
    if (!err) {
        const long long nLt = s_tot[0], Wt = s_tot[1], nLs = s_tot[2], Ws = s_tot[3];
        const long long nCt = (Wt + (1 << TL) - 1) >> TL, nCs = (Ws + (1 << SL) - 1) >> SL;
        const long long nwarps = (long long)G * NWF;
        const AV *val = (const AV *)a.val;
        const AV *sval = (const AV *)a.sval;
        for (long long ch = (long long)wid * G + b; ch < nCt + nCs; ch += nwarps) {
            if (ch < nCt) {
                // ---- tile chunk: 32 tile items, lane = item
                const long long base = ch << TL;
                FSTEP(0, 0);
                const long long s0 = __ldcg(&a.L.Ct[ch]);
                FSTEP(1, s0);
                const long long sq = s0 + lane;
                const bool inl = sq < nLt;
                const long long wq = inl ? __ldcg(&a.L.t_wpre[sq]) : INF64;
                const long long tbq = inl ? __ldcg(&a.L.t_beg[sq]) : 0;
                const unsigned xmq = inl ? __ldcg(&a.L.t_xm[sq]) : 0u;
                const int Jq = inl ? __ldcg(&a.L.t_J[sq]) : 0;
                FSTEP(2, wq + tbq + xmq + Jq);
                const long long d = wq - base;
                const unsigned starts = __reduce_or_sync(0xffffffffu, (lane > 0 && d > 0 && d < 32) ? 1u << d : 0u);
                const int qq = __popc(starts & (lane == 31 ? 0xffffffffu : ((2u << lane) - 1u)));
                const long long i = base + lane;
                const long long wsrc = __shfl_sync(0xffffffffu, wq, qq);
                const long long tbsrc = __shfl_sync(0xffffffffu, tbq, qq);
                const unsigned xm = __shfl_sync(0xffffffffu, xmq, qq);
                const int J = __shfl_sync(0xffffffffu, Jq, qq);
                const bool ok = i < Wt;
                const long long t = tbsrc + (i - wsrc);
                const unsigned hit = ok ? ((unsigned)__ldg(&a.mask[t]) & xm) : 0u;
                FSTEP(3, hit);
                TileRec16 r;
                r.off = 0;
                r.trow = 0;
                r.nnz = 0;
                r.b = make_uint4(0, 0, 0, 0);
                int useful = 0;
                if (hit) {
                    const uint4 *rp = reinterpret_cast<const uint4 *>(a.rec + t);
                    const uint4 h0 = __ldg(rp), h1 = __ldg(rp + 1);
                    r.off = h0.x;
                    r.trow = (int)h0.y;
                    r.nnz = h0.z;
                    r.b = h1;
                    useful = rec_useful(r.b, hit, (int)r.nnz);
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
                FSTEP(4, total);
                n_mac += useful;
                for (int q0 = 0; q0 < total; q0 += 32) {
                    const int qv = q0 + lane;
                    // source lane: smallest l with incl_l > qv
                    int lo = 0;
#pragma unroll
                    for (int step = 16; step >= 1; step >>= 1) {
                        const int v = __shfl_sync(0xffffffffu, incl, lo + step - 1);
                        if (v <= qv) lo += step;
                    }
                    lo = min(lo, 31);
                    const int exs = __shfl_sync(0xffffffffu, incl - useful, lo);
                    const unsigned off = __shfl_sync(0xffffffffu, r.off, lo);
                    const int trow = __shfl_sync(0xffffffffu, r.trow, lo);
                    const int nnz = __shfl_sync(0xffffffffu, (int)r.nnz, lo);
                    const unsigned hs = __shfl_sync(0xffffffffu, hit, lo);
                    const int Js = __shfl_sync(0xffffffffu, J, lo);
                    uint4 bs;
                    bs.x = __shfl_sync(0xffffffffu, r.b.x, lo);
                    bs.y = __shfl_sync(0xffffffffu, r.b.y, lo);
                    bs.z = __shfl_sync(0xffffffffu, r.b.z, lo);
                    bs.w = __shfl_sync(0xffffffffu, r.b.w, lo);
                    if (qv < total) {
                        int p, c, rr;
                        rec_position(bs, hs, nnz, qv - exs, p, c, rr);
                        const long long pos = (long long)off + p;
                        if (rr < 0) rr = __ldg(&a.idx[pos]) & (NT - 1);
                        const double av = val ? (double)__ldg(&val[pos]) : 1.0;
                        const double xv = __ldcg(&a.L.xd[(long long)Js * NT + c]);
                        const long long rc = trow >= 0 ? (long long)trow * NT + rr : ~((long long)(~trow) * NT + rr);
                        FSTEP(5, av + xv + rc);
                        contribute<SR>(a, s_hacc, s_hbits, rc, av, xv);
                    }
                }
                FSTEP(6, 0);
            } else {
                // ---- side chunk: 128 side nonzeros, window staged in shared memory
                const long long c2 = ch - nCt;
                const long long base = c2 << SL;
                const long long s0 = __ldcg(&a.L.Cs[c2]);
                long long *win = s_win + wid * WN;
                long long *winb = s_winb + wid * WN;
                double *winx = s_winx + wid * WN;
#pragma unroll
                for (int q0 = 0; q0 <= (1 << SL); q0 += 32) {
                    const int qx = q0 + lane;
                    const long long ix = s0 + qx;
                    const bool in = ix < nLs;
                    const long long w = in ? __ldcg(&a.L.s_wpre[ix]) : INF64;
                    const long long bg = in ? __ldcg(&a.L.s_beg[ix]) : 0;
                    const double xx = in ? __ldcg(&a.L.s_x[ix]) : 0.0;
                    if (qx <= (1 << SL)) {
                        win[qx] = w;
                        winb[qx] = bg;
                        winx[qx] = xx;
                    }
                }
                __syncwarp();
                ChunkMap<SL> cm;
                cm.build(win, base, lane);
                long long p[US];
                double xv[US];
                bool ok[US];
#pragma unroll
                for (int u = 0; u < US; ++u) {
                    const long long i = base + lane + 32 * u;
                    ok[u] = i < Ws;
                    const int qq = ok[u] ? cm.entry(lane + 32 * u) : 0;
                    p[u] = winb[qq] + (i - win[qq]);
                    xv[u] = winx[qq];
                }
                int row[US];
                double av[US];
#pragma unroll
                for (int u = 0; u < US; ++u) {
                    if (ok[u]) {
                        row[u] = __ldg(&a.srow[p[u]]);
                        av[u] = sval ? (double)__ldg(&sval[p[u]]) : 1.0;
                    }
                }
#pragma unroll
                for (int u = 0; u < US; ++u)
                    if (ok[u]) contribute<SR>(a, s_hacc, s_hbits, (long long)row[u], av[u], xv[u]);
                __syncwarp();
            }
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
    __syncthreads();
    // privatised hot rows: one global atomic per (CTA, touched hot row)
    if (!err) {
        for (int sl = tid; sl < n_slots; sl += FT) {
            if ((s_hbits[sl >> 5] >> (sl & 31)) & 1u) {
                const long long row = (long long)a.hot_list[sl / NT] * NT + sl % NT;
                if constexpr (SR == TSMV_PLUS_TIMES) atomicAdd(&a.acc[row], s_hacc[sl]);
                else if constexpr (SR == TSMV_MIN_SECOND)
                    atomicMax((unsigned long long *)&a.acc[row],
                              (unsigned long long)__double_as_longlong(s_hacc[sl]));
                atomicOr(&a.rowbits[row >> 5], 1u << (row & 31));
            }
        }
    }
    if (tid < 3) {
        long long sum = 0;
        for (int w = 0; w < NWF; ++w) sum += s_acct[w][tid];
        a.acct[b * 4 + tid] = sum;
    }
    grid_sync_f(&a.cnt->bar, target, tr ? tr + 3 : nullptr);
    if (stamp) ts[3] = globaltimer_ns();

    // ------------------------------------------------------------ phase C (a6)
    const long long S = (((a.W + G - 1) / G) + 31) & ~31ll;
    const long long w0 = (long long)b * S, w1 = min(a.W, w0 + S);
    long long mycnt = 0;
    for (long long w = w0 + tid; w < w1; w += FT) mycnt += __popc(__ldcg(&a.rowbits[w]));
    long long blk, dummy;
    block_scan<1, FT>(&mycnt, &dummy, &blk, s_scan);
    if (tid == 0) a.partials[b * 8 + 4] = blk;
    grid_sync_f(&a.cnt->bar, target, tr ? tr + 5 : nullptr);
    if (stamp) ts[4] = globaltimer_ns();
    if (tid < 32) {
        long long pre = 0, tt = 0;
        for (int g = lane; g < G; g += 32) {
            const long long v = __ldcg(&a.partials[g * 8 + 4]);
            tt += v;
            if (g < b) pre += v;
        }
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) {
            pre += __shfl_xor_sync(0xffffffffu, pre, o);
            tt += __shfl_xor_sync(0xffffffffu, tt, o);
        }
        if (lane == 0) {
            s_base[0] = pre;
            s_tot[0] = tt;
        }
    }
    __syncthreads();
    long long carry = s_base[0];
    const long long ycap = a.y_cap;
#ifdef TSMV_C2_DELAY
    { const unsigned long long t0 = globaltimer_ns(); while (globaltimer_ns() - t0 < 10000) {} }
#endif
    for (long long rb = w0; rb < w1; rb += FT) {
        const long long w = rb + tid;
        CSTEP(0, 0);
        const unsigned bits = w < w1 ? __ldcg(&a.rowbits[w]) : 0u;
        CSTEP(1, bits);
        long long c = __popc(bits), exw, rtot;
        block_scan<1, FT>(&c, &exw, &rtot, s_scan);
        CSTEP(2, exw);
        int it = 0;
        const long long pos0 = carry + exw;
        carry += rtot;
        if (bits) a.rowbits[w] = 0u;
        // transposed emission: the warp walks its words with bits, BATCH at a time;
        // lane l handles bit l of each, so acc loads and y stores are coalesced
        const long long wbase = w - lane;
        const unsigned lt = (1u << lane) - 1u;
        unsigned todo = __ballot_sync(0xffffffffu, bits != 0);
        while (todo) {
            int src[BATCH];
            int nb = 0;
#pragma unroll
            for (int kk = 0; kk < BATCH; ++kk) {
                src[kk] = 0;
                if (todo) {
                    src[kk] = __ffs(todo) - 1;
                    todo &= todo - 1;
                    nb = kk + 1;
                }
            }
            unsigned wb[BATCH];
            long long wp[BATCH];
            double v[BATCH];
            bool mine[BATCH];
#pragma unroll
            for (int kk = 0; kk < BATCH; ++kk) {
                wb[kk] = __shfl_sync(0xffffffffu, bits, src[kk]);
                wp[kk] = __shfl_sync(0xffffffffu, pos0, src[kk]);
                mine[kk] = kk < nb && ((wb[kk] >> lane) & 1u);
                if (mine[kk]) v[kk] = __ldcg(&a.acc[(wbase + src[kk]) * 32 + lane]);
            }
            CSTEP(3 + 2 * it, v[0] + v[BATCH - 1]);
#pragma unroll
            for (int kk = 0; kk < BATCH; ++kk) {
                if (mine[kk]) {
                    const long long row = (wbase + src[kk]) * 32 + lane;
                    const long long pos = wp[kk] + __popc(wb[kk] & lt);
#ifndef TSMV_C2_NOZERO
                    a.acc[row] = 0.0;
#endif
#ifdef TSMV_C2_NOSTORE
                    if (pos < 0) {
#else
                    if (pos < ycap) {
#endif
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
            CSTEP(4 + 2 * it, 0);
            ++it;
        }
    }
    if (b == 0 && tid == 0) {
        const long long yt = s_tot[0];
        a.cnt->y_nnz = yt;
        a.hm->y_nnz = yt;
        a.hm->err = err ? 1 : 0;
        if (a.ynnz_dev) *a.ynnz_dev = err ? -1 : yt;
        // every CTA read err / resv_* after barrier 1
        a.cnt->err = 0;
        a.cnt->resv_t = 0;
        a.cnt->resv_s = 0;
        if (a.tring) ts[5] = globaltimer_ns();
    }
    if (tr && tid == 0) tr[7] = globaltimer_ns();
}

template <class AV, class XV> void *pick_sr_flat(int sr) {
    if (sr == TSMV_PLUS_TIMES) return (void *)k_spmspv_flat<AV, XV, TSMV_PLUS_TIMES>;
    if (sr == TSMV_OR_AND) return (void *)k_spmspv_flat<AV, XV, TSMV_OR_AND>;
    return (void *)k_spmspv_flat<AV, XV, TSMV_MIN_SECOND>;
}
void *pick_flat(bool f32, int sr) { return f32 ? pick_sr_flat<float, float>(sr) : pick_sr_flat<double, double>(sr); }

constexpr size_t FLAT_DYN = HOT_SLOTS * 8 + (size_t)NWF * ((1 << SL) + 1) * 24 + HOT_SLOTS / 8;

void flat_set_smem() {
    static bool done = false;
    if (done) return;
    for (int f32 = 0; f32 < 2; ++f32)
        for (int sr = 0; sr < 3; ++sr)
            TSMV_CUDA(cudaFuncSetAttribute(pick_flat(f32, sr), cudaFuncAttributeMaxDynamicSharedMemorySize,
                                           (int)FLAT_DYN));
    done = true;
}

__global__ void k_build_rec16(const TileDesc *__restrict__ desc, const uint8_t *__restrict__ cstart,
                              const uint8_t *__restrict__ idx, int64_t T, TileRec16 *__restrict__ rec) {
    for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < T; t += (int64_t)gridDim.x * blockDim.x) {
        const TileDesc d = desc[t];
        TileRec16 r;
        r.off = (uint32_t)d.off;
        r.trow = d.trow;
        r.nnz = (uint32_t)d.nnz;
        r.pad = 0;
        uint8_t by[16];
        for (int i = 0; i < 16; ++i) by[i] = d.nnz <= 16 ? (i < d.nnz ? idx[d.off + i] : 0xffu) : cstart[t * 16 + i];
        r.b.x = by[0] | (by[1] << 8) | (by[2] << 16) | ((unsigned)by[3] << 24);
        r.b.y = by[4] | (by[5] << 8) | (by[6] << 16) | ((unsigned)by[7] << 24);
        r.b.z = by[8] | (by[9] << 8) | (by[10] << 16) | ((unsigned)by[11] << 24);
        r.b.w = by[12] | (by[13] << 8) | (by[14] << 16) | ((unsigned)by[15] << 24);
        rec[t] = r;
    }
}

}  // namespace

bool flat_supported(const tsmv_ctx *c) {
    return c->nt == 16 && c->P.rec.p != nullptr && !getenv("TSMV_FUSED_V6");
}

void build_rec16(tsmv_ctx *c, TileSet &S, cudaStream_t st) {
    if (c->nt != 16 || S.T == 0 || S.dense_nnz >= (1ll << 32)) return;
    S.rec.alloc((size_t)S.T * sizeof(TileRec16));
    const int blocks = (int)std::min<int64_t>((S.T + 255) / 256, 148 * 16);
    k_build_rec16<<<blocks, 256, 0, st>>>(S.desc.as<TileDesc>(), S.cstart.as<uint8_t>(), S.idx.as<uint8_t>(), S.T,
                                          S.rec.as<TileRec16>());
    TSMV_CUDA(cudaGetLastError());
}

int flat_occupancy(int dtype) {
    int bps = 0;
    flat_set_smem();
    void *f = pick_flat(dtype == TSMV_F32, TSMV_PLUS_TIMES);
    cudaError_t e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&bps, f, FT, FLAT_DYN);
    if (e != cudaSuccess) {
        cudaGetLastError();
        bps = 0;
    }
    return bps;
}

void ensure_flat_lists(tsmv_ctx *c, int64_t k) {
    FlatLists &F = c->FL;
    if (k > F.cap_ent) {
        const int64_t cap = std::max<int64_t>(k, 1024);
        const int64_t segs = std::min<int64_t>(cap, c->nTC) + 1;
        F.t_beg.alloc(segs * 8);
        F.t_wpre.alloc(segs * 8);
        F.t_xm.alloc(segs * 4);
        F.t_J.alloc(segs * 4);
        F.s_beg.alloc((cap + 1) * 8);
        F.s_wpre.alloc((cap + 1) * 8);
        F.s_x.alloc((cap + 1) * 8);
        F.cap_ent = cap;
    }
    if (!F.Ct.p) {
        F.Ct.alloc(((c->P.T >> TL) + 2) * 4);
        F.Cs.alloc(((c->P.side_nnz >> SL) + 2) * 4);
    }
}

FlatListsView flat_view(tsmv_ctx *c) {
    FlatListsView v;
    v.t_beg = c->FL.t_beg.as<long long>();
    v.t_wpre = c->FL.t_wpre.as<long long>();
    v.t_xm = c->FL.t_xm.as<unsigned>();
    v.t_J = c->FL.t_J.as<int>();
    v.s_beg = c->FL.s_beg.as<long long>();
    v.s_wpre = c->FL.s_wpre.as<long long>();
    v.s_x = c->FL.s_x.as<double>();
    v.Ct = c->FL.Ct.as<int>();
    v.Cs = c->FL.Cs.as<int>();
    v.xd = c->xdense.as<double>();
    return v;
}

// Enqueue one flat SpMSpV (device pointers only, no sync).  Returns false if the
// context cannot use it (nt != 16).
void enqueue_spmspv_flat(tsmv_ctx *c, int sr, long long k, const int32_t *xi, const void *xv, long long ycap,
                         int32_t *yi, void *yv, long long *ynnz_dev, cudaStream_t st) {
    const bool f32 = c->dtype == TSMV_F32;
    ensure_flat_lists(c, k);
    FlatArgs a;
    a.x_idx = xi;
    a.x_val = xv;
    a.k = k;
    a.n = c->n;
    a.m = c->m;
    a.W = (c->m + 31) / 32;
    a.row_begin = c->row_begin;
    a.tptr = c->P.ptr.as<long long>();
    a.mask = c->P.mask.as<uint16_t>();
    a.rec = c->P.rec.as<TileRec16>();
    a.idx = c->P.idx.as<uint8_t>();
    a.val = c->P.has_vals ? c->P.val.p : nullptr;
    a.sptr = c->P.sptr.as<long long>();
    a.srow = c->P.srow.as<int>();
    a.sval = c->P.has_vals ? c->P.sval.p : nullptr;
    a.L = flat_view(c);
    a.acc = c->acc.as<double>();
    a.rowbits = c->rowbits_p;
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
    a.hot_list = c->P.hot_list;
    a.n_hot = c->P.hot_list ? c->n_hot : 0;
    a.trace = (unsigned long long *)c->trace;
    void *args[] = {&a};
    const int G = c->flat_blocks;
    flat_set_smem();
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(G);
    cfg.blockDim = dim3(FT);
    cfg.dynamicSmemBytes = FLAT_DYN;
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
    TSMV_CUDA(cudaLaunchKernelExC(&cfg, pick_flat(f32, sr), args));
    c->bar_base += 3ull * (unsigned long long)G;
    c->last_blocks = G;
    if (c->timing) c->tcalls++;
}

}  // namespace tsmv
