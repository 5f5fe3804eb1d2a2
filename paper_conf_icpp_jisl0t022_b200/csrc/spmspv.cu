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
#include <cub/device/device_radix_sort.cuh>

namespace tsmv {

namespace {

#ifndef TSMV_FB
#define TSMV_FB 512
#endif
#ifndef TSMV_CB
#define TSMV_CB 8
#endif
constexpr int FB = TSMV_FB;  // threads per CTA of the fused kernel
constexpr int CB = TSMV_CB;  // accumulator loads batched per lane in phase C
#ifndef TSMV_R
#define TSMV_R 2
#endif
#ifndef TSMV_SCL
#define TSMV_SCL 7
#endif
constexpr int R = TSMV_R;     // useful nonzeros per lane per round of the multiply step
constexpr int SCL = TSMV_SCL; // log2 of the items per warp-chunk of the SpMSpV load balancer
constexpr int SCH = 1 << SCL;
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
    const int32_t *hot_list;    // privatised tile rows (TileSet::hot_list), n_hot of them
    int n_hot;
    unsigned long long *trace;  // tsmv_set_trace: per warp {t_B0, t_loop_end, chunks, tile ns, side ns, max chunk ns, t_arrive, macs}
};

#ifdef TSMV_TRACE_STEPS
// development: stamp step k of the warp that processes tile chunk 0 (after a fake
// use of `dep` so the stamp waits for the loads that produced it)
#define STEP(k, dep)                                                                          \
    do {                                                                                      \
        if (a.trace && ch == 0 && lane == 0) {                                                \
            if ((long long)(dep) == 0x5eed5eed5eedll) a.trace[1000] = 1;                     \
            a.trace[200 + (k)] = globaltimer_ns();                                            \
        }                                                                                     \
    } while (0)
#else
#define STEP(k, dep) ((void)0)
#endif

#ifdef TSMV_EXPERIMENT_NO_ROWBITS
#define TOUCH(p, b) ((void)0)  // timing experiment only: y comes out empty
#else
#define TOUCH(p, b) atomicOr((p), (b))
#endif

// Shared-memory accumulation of the privatised ("hot") rows.
template <int SR>
__device__ __forceinline__ void accumulate_shared(double *s_acc, long long slot, double a, double x) {
    if constexpr (SR == TSMV_PLUS_TIMES) {
        atomicAdd(&s_acc[slot], a * x);
    } else if constexpr (SR == TSMV_MIN_SECOND) {
        atomicMax((unsigned long long *)&s_acc[slot], ~ord_key(x));
    }
}

template <int SR>
__device__ __forceinline__ void accumulate_value(double *acc, long long row, double a, double x) {
    if constexpr (SR == TSMV_PLUS_TIMES) {
#ifdef TSMV_EXPERIMENT_NO_ATOMIC
        if (a * x == 1234.5678) acc[row] = 0.0;  // keeps the loads, drops the RED
#else
        atomicAdd(&acc[row], a * x);
#endif
    } else if constexpr (SR == TSMV_MIN_SECOND) {
        atomicMax((unsigned long long *)&acc[row], ~ord_key(x));
    }
}

// Touched-row bits of rows rowbase + {bits of m} (rowbase is a multiple of NT, so
// the rows of one tile share a word, or two for NT = 64).  Test before set:
// power-law rows receive thousands of contributions per call and an
// unconditional RED.OR on their shared word serialises in one L2 slice; the L1
// copy can only be stale towards "not set", which costs a redundant RED.
template <int NT>
__device__ __forceinline__ void mark_rows(uint32_t *rowbits, long long rowbase, typename Tr<NT>::word_t m) {
    if constexpr (NT == 64) {
        uint32_t lo = (uint32_t)m, hi = (uint32_t)((unsigned long long)m >> 32);
        uint32_t *w = rowbits + (rowbase >> 5);
        if (lo && (__ldca(w) & lo) != lo) atomicOr(w, lo);
        if (hi && (__ldca(w + 1) & hi) != hi) atomicOr(w + 1, hi);
    } else {
        const uint32_t b = (uint32_t)m << (rowbase & 31);
        uint32_t *w = rowbits + (rowbase >> 5);
        if ((__ldca(w) & b) != b) atomicOr(w, b);
    }
}

template <int NT>
__device__ __forceinline__ void mark_rows_shared(uint32_t *s_bits, long long slotbase, typename Tr<NT>::word_t m) {
    if constexpr (NT == 64) {
        atomicOr(&s_bits[slotbase >> 5], (uint32_t)m);
        atomicOr(&s_bits[(slotbase >> 5) + 1], (uint32_t)((unsigned long long)m >> 32));
    } else {
        atomicOr(&s_bits[slotbase >> 5], (uint32_t)m << (slotbase & 31));
    }
}

// Staged hit tile of one lane (multiply step of phase B).
struct Stage {
    long long off, t;
    unsigned long long hit;
    int incl, J, trow, nnz;
};

// Column range [p0, p1) of column c inside tile t (column-major nonzeros).
template <int NT>
__device__ __forceinline__ void col_range(const typename Tr<NT>::cs_t *cstart, long long t, int c, int nnz, int &p0,
                                          int &p1) {
    p0 = cstart[t * NT + c];
    p1 = c + 1 < NT ? (int)cstart[t * NT + c + 1] : nnz;
}

// nt = 16: the 16 one-byte column starts of a tile are one aligned 16-byte
// load; the column walks below then run in registers (a walk over global
// memory is a chain of dependent L2 round trips, ~1 us per hit column).
__device__ __forceinline__ uint4 cs_row16(const uint8_t *cstart, long long t) {
    return __ldg(reinterpret_cast<const uint4 *>(cstart + t * 16));
}
__device__ __forceinline__ int cs_byte16(const uint4 &w, int c, int nnz) {
    if (c >= 16) return nnz;
    const unsigned x = c < 8 ? (c < 4 ? w.x : w.y) : (c < 12 ? w.z : w.w);
    return (int)((x >> ((c & 3) * 8)) & 0xffu);
}

__device__ __forceinline__ int hit_useful16(const uint4 &w, unsigned h, int nnz) {
    int s = 0;
    while (h) {
        const int c = __ffs(h) - 1;
        h &= h - 1;
        s += cs_byte16(w, c + 1, nnz) - cs_byte16(w, c, nnz);
    }
    return s;
}
__device__ __forceinline__ void hit_position16(const uint4 &w, unsigned h, int nnz, int k, int &c, int &p) {
    c = 0;
    p = 0;
    while (h) {
        c = __ffs(h) - 1;
        h &= h - 1;
        const int p0 = cs_byte16(w, c, nnz), len = cs_byte16(w, c + 1, nnz) - p0;
        if (k < len) {
            p = p0 + k;
            return;
        }
        k -= len;
    }
}

// Useful nonzeros of a hit tile = sum over its hit columns of the column lengths.
template <int NT>
__device__ __forceinline__ int hit_useful(const typename Tr<NT>::cs_t *cstart, long long t,
                                          typename Tr<NT>::word_t h, int nnz) {
    if constexpr (NT == 16) {
        const uint4 w = cs_row16((const uint8_t *)cstart, t);
        int s = 0;
        while (h) {
            const int c = ffs_w(h);
            h &= h - 1;
            s += cs_byte16(w, c + 1, nnz) - cs_byte16(w, c, nnz);
        }
        return s;
    }
    int s = 0;
    while (h) {
        const int c = ffs_w(h);
        h &= h - 1;
        int p0, p1;
        col_range<NT>(cstart, t, c, nnz, p0, p1);
        s += p1 - p0;
    }
    return s;
}

// The k-th useful nonzero of a hit tile: its column c and position p in the tile.
template <int NT>
__device__ __forceinline__ void hit_position(const typename Tr<NT>::cs_t *cstart, long long t,
                                             typename Tr<NT>::word_t h, int nnz, int k, int &c, int &p) {
    c = 0;
    p = 0;
    if constexpr (NT == 16) {
        const uint4 w = cs_row16((const uint8_t *)cstart, t);
        while (h) {
            c = ffs_w(h);
            h &= h - 1;
            const int p0 = cs_byte16(w, c, nnz), len = cs_byte16(w, c + 1, nnz) - p0;
            if (k < len) {
                p = p0 + k;
                return;
            }
            k -= len;
        }
        return;
    }
    while (h) {
        c = ffs_w(h);
        h &= h - 1;
        int p0, p1;
        col_range<NT>(cstart, t, c, nnz, p0, p1);
        if (k < p1 - p0) {
            p = p0 + k;
            return;
        }
        k -= p1 - p0;
    }
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
    constexpr int U = SCH / 32;
    constexpr int NW = FB / 32;
    __shared__ long long s_scan[8][NW];  // block_scan scratch (K prefixes + K totals)
    __shared__ long long win_all[NW][SCH + 1];

    __shared__ long long s_pre[4], s_tot[4];
    __shared__ long long s_acct[NW][3];
    __shared__ int s_err;
    extern __shared__ __align__(16) unsigned char s_dyn[];
    double *s_hacc = reinterpret_cast<double *>(s_dyn);                   // [HOT_SLOTS]
    uint32_t *s_hbits = reinterpret_cast<uint32_t *>(s_dyn + HOT_SLOTS * 8);  // [HOT_SLOTS/32]
    Stage *stage_all = reinterpret_cast<Stage *>(s_dyn + HOT_SLOTS * 8 + HOT_SLOTS / 8);  // [NW][SCH]
    long long *win_b = reinterpret_cast<long long *>(stage_all + NW * SCH);                // [NW][SCH+1]
    double *win_x = reinterpret_cast<double *>(win_b + NW * (SCH + 1));                    // [NW][SCH+1]
    const int n_slots = a.n_hot * NT;
    const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
    const int G = gridDim.x, b = blockIdx.x;
    unsigned long long target = a.bar_base;
    const bool stamp = a.tring && b == 0 && tid == 0;
    unsigned long long *ts_out = a.tring ? a.tring + (a.tslot % TRING) * 8 : nullptr;
    if (stamp) ts_out[0] = globaltimer_ns();

    for (int i = tid; i < n_slots; i += FB) s_hacc[i] = 0.0;
    for (int i = tid; i < (n_slots + 31) / 32; i += FB) s_hbits[i] = 0u;

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
    block_scan<4, FB>(q.v, ex.v, agg.v, s_scan);
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
                write_chunks<SCL>(a.Lv.Ct, oWt, wt, (int)oLt);
                ++oLt;
                oWt += wt;
            }
            if (ws > 0) {
                a.Lv.Ls_beg[oLs] = a.sptr[j];
                a.Lv.Ls_wpre[oLs] = oWs;
                a.Lv.Ls_x[oLs] = a.x_val ? (double)((const XV *)a.x_val)[e] : 1.0;
                write_chunks<SCL>(a.Lv.Cs, oWs, ws, (int)oLs);
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
        const long long nCt = (Wt + SCH - 1) >> SCL, nCs = (Ws + SCH - 1) >> SCL;
        long long *win = win_all[wid];
        const word_t *mask = (const word_t *)a.mask;
        const idx_t *idx = (const idx_t *)a.idx;
        const AV *val = (const AV *)a.val;
        const AV *sval = (const AV *)a.sval;
        const cs_t *cstart = (const cs_t *)a.cstart;
        const unsigned nwarps = (unsigned)(G * NW);
        unsigned ch = (unsigned)(b * NW + wid);  // first chunk static, then the queue
        unsigned long long tr_b0 = 0, tr_tile = 0, tr_side = 0, tr_max = 0, tr_n = 0, tr_stage = 0, tr_smax = 0;
#ifdef TSMV_TRACE_ROUNDS
        unsigned long long tr_pos = 0, tr_ld = 0, tr_at = 0;
#endif
        if (a.trace) tr_b0 = globaltimer_ns();
        while (true) {
            const unsigned long long tr_c0 = a.trace ? globaltimer_ns() : 0;
            const bool tr_is_tile = ch < nCt;
            // grab the next chunk now; its latency overlaps this chunk's work
            unsigned nx = 0;
            if (lane == 0 && ch < nCt + nCs) nx = nwarps + atomicAdd(&a.cnt->chunk_next, 1u);
            if (ch < nCt) {
                STEP(0, 0);
                const long long s0 = __ldcg(&a.Lv.Ct[ch]);
                STEP(1, s0);
                const long long base = (long long)ch << SCL;
                load_window<SCL>(win, a.Lv.Lt_wpre, s0, nLt, lane);
                STEP(2, win[0]);
                long long sidx[U], t[U];
                bool ok[U];
                ChunkMap<SCL> cm;
                cm.build(win, base, lane);
#pragma unroll
                for (int u = 0; u < U; ++u) {
                    const long long i = base + lane + 32 * u;
                    ok[u] = i < Wt;
                    const int qq = ok[u] ? cm.entry(lane + 32 * u) : 0;
                    sidx[u] = s0 + qq;
                    t[u] = i - win[qq];
                }
                STEP(3, sidx[0] + t[0]);
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
                STEP(4, t[0] + xm[0] + J[0]);
                word_t hit[U];
#pragma unroll
                for (int u = 0; u < U; ++u) hit[u] = ok[u] ? (word_t)(mask[t[u]] & xm[u]) : (word_t)0;
                // ---- multiply: nonzero-level load balance inside the warp.  The hit
                // tiles of all U items of all lanes are staged in shared memory with the
                // inclusive prefix of their useful nonzeros (sum over hit columns); the
                // warp then walks that flat index space R positions per lane at a time,
                // so a dense hub tile is spread over the warp and the loads of different
                // positions are issued together.
                STEP(5, hit[0] + hit[1]);
                TileDesc d[U];
#pragma unroll
                for (int u = 0; u < U; ++u)
                    if (hit[u]) d[u] = ((const TileDesc *)a.desc)[t[u]];
                STEP(6, d[0].off + d[1].off);
                int useful[U];
                int mine = 0;
                uint4 csr[U];
                if constexpr (NT == 16) {
#pragma unroll
                    for (int u = 0; u < U; ++u)
                        if (hit[u]) csr[u] = cs_row16((const uint8_t *)cstart, t[u]);
                }
#pragma unroll
                for (int u = 0; u < U; ++u) {
                    if constexpr (NT == 16)
                        useful[u] = hit[u] ? hit_useful16(csr[u], (unsigned)hit[u], d[u].nnz) : 0;
                    else
                        useful[u] = hit[u] ? hit_useful<NT>(cstart, t[u], hit[u], d[u].nnz) : 0;
                    mine += useful[u];
                    if (hit[u]) {
                        ++n_hit;
                        n_hcol += popc_w(hit[u]);
                    }
                }
                STEP(7, mine);
                n_mac += mine;
                int incl = mine;
#pragma unroll
                for (int o = 1; o < 32; o <<= 1) {
                    const int v = __shfl_up_sync(0xffffffffu, incl, o);
                    if (lane >= o) incl += v;
                }
                const int total = __shfl_sync(0xffffffffu, incl, 31);
                if (a.trace) tr_stage = globaltimer_ns() - tr_c0;
                STEP(8, total);
                if (total > 0) {
                    Stage *st = stage_all + wid * SCH;
                    int run = incl - mine;
#pragma unroll
                    for (int u = 0; u < U; ++u) {
                        run += useful[u];
                        Stage &sg = st[lane * U + u];
                        sg.incl = run;
                        if (useful[u]) {
                            sg.t = t[u];
                            sg.J = (int)J[u];
                            sg.off = d[u].off;
                            sg.hit = (unsigned long long)hit[u];
                            sg.trow = d[u].trow;
                            sg.nnz = d[u].nnz;
                        }
                    }
                    __syncwarp();
                    STEP(9, 0);
                    for (int q0 = 0; q0 < total; q0 += 32 * R) {
#ifdef TSMV_TRACE_ROUNDS
                        const unsigned long long rt0 = globaltimer_ns();
#endif
                        long long row[R], pos[R], xj[R];
                        bool okq[R], hot[R];
                        int srcq[R], kq[R];
#pragma unroll
                        for (int r = 0; r < R; ++r) {
                            const int q = q0 + 32 * r + lane;
                            okq[r] = q < total;
                            srcq[r] = 0;
                            kq[r] = 0;
                            if (okq[r]) {
                                int lo = 0, hi = SCH - 1;  // first staged entry with incl > q
                                while (lo < hi) {
                                    const int mid = (lo + hi) >> 1;
                                    if (st[mid].incl > q) hi = mid;
                                    else lo = mid + 1;
                                }
                                srcq[r] = lo;
                                kq[r] = q - (lo ? st[lo - 1].incl : 0);
                            }
                        }
                        uint4 cq[R];
                        if constexpr (NT == 16) {
#pragma unroll
                            for (int r = 0; r < R; ++r)
                                if (okq[r]) cq[r] = cs_row16((const uint8_t *)cstart, st[srcq[r]].t);
                        }
#pragma unroll
                        for (int r = 0; r < R; ++r) {
                            if (okq[r]) {
                                const Stage &src = st[srcq[r]];
                                int c, p;
                                if constexpr (NT == 16)
                                    hit_position16(cq[r], (unsigned)src.hit, src.nnz, kq[r], c, p);
                                else
                                    hit_position<NT>(cstart, src.t, (word_t)src.hit, src.nnz, kq[r], c, p);
                                hot[r] = src.trow < 0;
                                row[r] = (hot[r] ? (long long)(~src.trow) : (long long)src.trow) * NT;
                                pos[r] = src.off + p;
                                xj[r] = (long long)src.J * NT + c;
                            }
                        }
                        STEP(10, pos[0] + row[0]);
                        double av[R], xv[R];
#ifdef TSMV_TRACE_ROUNDS
                        __syncwarp();
                        const unsigned long long rt1 = globaltimer_ns();
#endif
#pragma unroll
                        for (int r = 0; r < R; ++r) {
                            if (okq[r]) {
                                row[r] += idx[pos[r]] & (NT - 1);
                                av[r] = val ? (double)val[pos[r]] : 1.0;
                                xv[r] = __ldcg(&a.Lv.xd[xj[r]]);
                            }
                        }
                        STEP(11, (long long)(av[0] + xv[0]) + row[0]);
#ifdef TSMV_TRACE_ROUNDS
                        {
                            double sink = 0;
                            for (int r = 0; r < R; ++r) if (okq[r]) sink += av[r] + xv[r] + (double)row[r];
                            if (sink == 1.2345e300) a.acc[0] = sink;
                        }
                        __syncwarp();
                        const unsigned long long rt2 = globaltimer_ns();
#endif
#pragma unroll
                        for (int r = 0; r < R; ++r) {
                            if (okq[r]) {
                                if (hot[r]) {
                                    accumulate_shared<SR>(s_hacc, row[r], av[r], xv[r]);
                                    atomicOr(&s_hbits[row[r] >> 5], 1u << (row[r] & 31));
                                } else {
                                    accumulate_value<SR>(a.acc, row[r], av[r], xv[r]);
                                }
                            }
                        }
                        // touched bit: rows of hub tile rows are privatised (shared memory),
                        // so the remaining RED.ORs are spread over many words -> no test load
#pragma unroll
                        for (int r = 0; r < R; ++r)
                            if (okq[r] && !hot[r]) TOUCH(&a.rowbits[row[r] >> 5], 1u << (row[r] & 31));
                        STEP(12, 0);
#ifdef TSMV_TRACE_ROUNDS
                        __syncwarp();
                        const unsigned long long rt3 = globaltimer_ns();
                        tr_pos += rt1 - rt0;
                        tr_ld += rt2 - rt1;
                        tr_at += rt3 - rt2;
#endif
                    }
                    __syncwarp();
                }
            } else if (ch < nCt + nCs) {
                const long long c2 = (long long)ch - nCt;
                const long long s0 = __ldcg(&a.Lv.Cs[c2]);
                const long long base = c2 << SCL;
                // window of the side list with its payload (column start, x_j) in shared
                // memory: one coalesced load phase instead of a dependent hop per item
                long long *winb = win_b + wid * (SCH + 1);
                double *winx = win_x + wid * (SCH + 1);
#pragma unroll
                for (int q0 = 0; q0 <= SCH; q0 += 32) {
                    const int q = q0 + lane;
                    const long long ix = s0 + q;
                    const bool in = ix <= nLs;
                    const long long w = in ? __ldcg(&a.Lv.Ls_wpre[ix]) : 0x7fffffffffffffffLL;
                    const long long bg = (in && ix < nLs) ? __ldcg(&a.Lv.Ls_beg[ix]) : 0;
                    const double xx = (in && ix < nLs) ? __ldcg(&a.Lv.Ls_x[ix]) : 0.0;
                    if (q <= SCH) {
                        win[q] = w;
                        winb[q] = bg;
                        winx[q] = xx;
                    }
                }
                __syncwarp();
                long long p[U];
                double xv[U];
                bool ok[U];
                ChunkMap<SCL> cm;
                cm.build(win, base, lane);
#pragma unroll
                for (int u = 0; u < U; ++u) {
                    const long long i = base + lane + 32 * u;
                    ok[u] = i < Ws;
                    const int qq = ok[u] ? cm.entry(lane + 32 * u) : 0;
                    p[u] = winb[qq] + (i - win[qq]);
                    xv[u] = winx[qq];
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
                for (int u = 0; u < U; ++u) {
                    if (ok[u] && row[u] < 0) {  // privatised row: shared memory
                        const long long sl = ~row[u];
                        accumulate_shared<SR>(s_hacc, sl, av[u], xv[u]);
                        atomicOr(&s_hbits[sl >> 5], 1u << (sl & 31));
                        ok[u] = false;
                    }
                }
#pragma unroll
                for (int u = 0; u < U; ++u)
                    if (ok[u]) accumulate_value<SR>(a.acc, row[u], av[u], xv[u]);
#pragma unroll
                for (int u = 0; u < U; ++u)
                    if (ok[u]) TOUCH(&a.rowbits[row[u] >> 5], 1u << (row[u] & 31));
            } else {
                break;
            }
            __syncwarp();
            if (a.trace) {
                const unsigned long long dt = globaltimer_ns() - tr_c0;
                (tr_is_tile ? tr_tile : tr_side) += dt;
                if (dt > tr_max) tr_smax = tr_is_tile ? tr_stage : 0;
                tr_max = dt > tr_max ? dt : tr_max;
                ++tr_n;
            }
            ch = __shfl_sync(0xffffffffu, nx, 0);
        }
        if (a.trace && lane == 0) {
            unsigned long long *tw = a.trace + ((long long)b * NW + wid) * 8;
            tw[0] = tr_b0;
            tw[1] = globaltimer_ns();
            tw[2] = tr_n;
            tw[3] = tr_tile;
            tw[4] = tr_side;
            tw[5] = tr_max;
            tw[6] = tr_smax;
#ifdef TSMV_TRACE_ROUNDS
            tw[3] = tr_pos;
            tw[4] = tr_ld;
            tw[6] = tr_at;
#endif
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
    // flush the privatised rows: one global atomic per (CTA, touched hot row)
    __syncthreads();
    if (!err) {
        for (int sl = tid; sl < n_slots; sl += FB) {
            if ((s_hbits[sl >> 5] >> (sl & 31)) & 1u) {
                const long long row = (long long)a.hot_list[sl / NT] * NT + sl % NT;
                if constexpr (SR == TSMV_PLUS_TIMES) atomicAdd(&a.acc[row], s_hacc[sl]);
                else if constexpr (SR == TSMV_MIN_SECOND)
                    atomicMax((unsigned long long *)&a.acc[row], (unsigned long long)__double_as_longlong(s_hacc[sl]));
                const unsigned bit = 1u << (row & 31);
                if (!(__ldca(&a.rowbits[row >> 5]) & bit)) atomicOr(&a.rowbits[row >> 5], bit);
            }
        }
    }
    if (a.trace && lane == 0) {
        unsigned long long *tw = a.trace + ((long long)b * NW + wid) * 8;
        tw[7] = (unsigned long long)n_mac;
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
        block_scan<1, FB>(&mycnt, &dummy, &blk, s_scan);
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
        block_scan<1, FB>(&c, &exw, &rtot, s_scan);
        const long long pos0 = carry + exw;
        carry += rtot;
        if (bits) a.rowbits[w] = 0u;
        const long long wbase = w - lane;
        unsigned todo = __ballot_sync(0xffffffffu, bits != 0);
        while (todo) {
            int src[CB];
            int nb = 0;
#pragma unroll
            for (int kk = 0; kk < CB; ++kk) {
                src[kk] = 0;
                if (todo) {
                    src[kk] = __ffs(todo) - 1;
                    todo &= todo - 1;
                    nb = kk + 1;
                }
            }
            unsigned wb[CB];
            long long wp[CB];
            double v[CB];
            bool mine[CB];
#pragma unroll
            for (int kk = 0; kk < CB; ++kk) {
                wb[kk] = __shfl_sync(0xffffffffu, bits, src[kk]);
                wp[kk] = __shfl_sync(0xffffffffu, pos0, src[kk]);
                mine[kk] = kk < nb && ((wb[kk] >> lane) & 1u);
                if (mine[kk]) v[kk] = __ldcg(&a.acc[(wbase + src[kk]) * 32 + lane]);
            }
#pragma unroll
            for (int kk = 0; kk < CB; ++kk) {
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
        __syncthreads();  // s_scan reuse
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

size_t fused_dyn_smem() {
    return HOT_SLOTS * 8 + HOT_SLOTS / 8 + (size_t)(FB / 32) * SCH * sizeof(Stage) + (size_t)(FB / 32) * (SCH + 1) * 16;
}

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
    const size_t dyn = fused_dyn_smem();
    cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)dyn);
    cudaError_t e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&bps, f, FB, dyn);
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
        int64_t nct = (c->P.T + SCH - 1) / SCH + 2;
        int64_t ncs = (c->P.side_nnz + SCH - 1) / SCH + 2;
        L.Ct.alloc(nct * 4);
        L.Cs.alloc(ncs * 4);
        L.cap_ct = nct;
        L.cap_cs = ncs;
    }
}

// Enqueue one fused SpMSpV (device pointers only, no sync).
void enqueue_spmspv(tsmv_ctx *c, int sr, long long k, const int32_t *xi, const void *xv, long long ycap,
                    int32_t *yi, void *yv, long long *ynnz_dev, cudaStream_t st) {
    if (use_rows_kernel(c, k)) {
        ensure_flat_lists(c, k);  // piece-count buffers shared with the flat kernel
        enqueue_spmspv_rows(c, sr, k, xi, xv, ycap, yi, yv, ynnz_dev, st);
        return;
    }
    if (flat_supported(c)) {
        enqueue_spmspv_flat(c, sr, k, xi, xv, ycap, yi, yv, ynnz_dev, st);
        return;
    }
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
    void *f = pick_kernel(c->nt, f32, sr);
    const size_t dyn = fused_dyn_smem();
    TSMV_CUDA(cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)dyn));
    TSMV_CUDA(cudaLaunchCooperativeKernel(f, dim3(c->fused_blocks), dim3(FB), args, dyn, st));
    c->bar_base += 4ull * (unsigned long long)c->fused_blocks;
    c->last_blocks = c->fused_blocks;
    if (c->timing) c->tcalls++;
}

void stats_from_partials(tsmv_ctx *c, tsmv_call_stats *s) {
    const int G = c->last_blocks;
    std::vector<long long> p(8 * (size_t)G), q(4 * (size_t)G);
    TSMV_CUDA(cudaMemcpy(p.data(), c->partials.p, p.size() * 8, cudaMemcpyDeviceToHost));
    TSMV_CUDA(cudaMemcpy(q.data(), c->acct.p, q.size() * 8, cudaMemcpyDeviceToHost));
    s->x_segments = s->tile_items = s->side_items = 0;
    s->hit_tiles = s->hit_columns = s->tile_macs = s->tile_macs_indirect = 0;
    long long nLs = 0;
    for (int b = 0; b < G; ++b) {
        s->x_segments += p[8 * b];
        s->tile_items += p[8 * b + 1];
        nLs += p[8 * b + 2];
        s->side_items += p[8 * b + 3];
        s->hit_tiles += q[4 * b];
        s->hit_columns += q[4 * b + 1];
        s->tile_macs += q[4 * b + 2];
        s->tile_macs_indirect += (c->use_flat ? q[4 * b + 3] : q[4 * b + 2]);
    }
    (void)nLs;
}

}  // namespace tsmv

using namespace tsmv;

namespace tsmv {
namespace {
// y (device staging) -> caller's pinned host y, sized on the device by the
// call's y_nnz (no host round trip between the multiply and the copy):
// 16-byte stores where both sides are aligned, full PCIe write lines.
__global__ void k_copy_y(const int32_t *__restrict__ yi, const void *__restrict__ yv, const long long *__restrict__ ynnz,
                         long long ycap, int32_t *__restrict__ hyi, void *__restrict__ hyv, int vb) {
    const long long n = min(*ynnz, ycap);
    const long long tid = blockIdx.x * (long long)blockDim.x + threadIdx.x, nt = (long long)gridDim.x * blockDim.x;
    if (hyi) {
        const bool al = ((reinterpret_cast<uintptr_t>(hyi) & 15) == 0);
        const long long nv = al ? n / 4 : 0;
        for (long long i = tid; i < nv; i += nt)
            reinterpret_cast<int4 *>(hyi)[i] = __ldcg(reinterpret_cast<const int4 *>(yi) + i);
        for (long long i = nv * 4 + tid; i < n; i += nt) hyi[i] = yi[i];
    }
    if (hyv) {
        const long long bytes = n * vb;
        const bool al = ((reinterpret_cast<uintptr_t>(hyv) & 15) == 0);
        const long long nv = al ? bytes / 16 : 0;
        for (long long i = tid; i < nv; i += nt)
            reinterpret_cast<int4 *>(hyv)[i] = __ldcg(reinterpret_cast<const int4 *>(yv) + i);
        for (long long i = nv * 16 + tid; i < bytes; i += nt)
            static_cast<char *>(hyv)[i] = static_cast<const char *>(yv)[i];
    }
}
}  // namespace
}  // namespace tsmv

// Reading R21: x in any order of unique indices.  The kernels take ascending x
// (segments are runs); an x they reject is sorted here once (CUB radix sort of
// (index, value) pairs into ctx buffers) and the call is repeated; duplicates
// or out-of-range indices are then still rejected (EINVAL).
static void sort_x(tsmv_ctx *c, long long k, const int32_t *xi, const void *xv, size_t vb, const int32_t **xi_out,
                   const void **xv_out, cudaStream_t st) {
    c->sort_x_idx.ensure((size_t)k * 4);
    if (xv) c->sort_x_val.ensure((size_t)k * vb);
    int32_t *ko = c->sort_x_idx.as<int32_t>();
    size_t tb = 0;
    if (!xv) {
        TSMV_CUDA(cub::DeviceRadixSort::SortKeys(nullptr, tb, xi, ko, (int)k, 0, 32, st));
        c->sort_tmp.ensure(tb);
        TSMV_CUDA(cub::DeviceRadixSort::SortKeys(c->sort_tmp.p, tb, xi, ko, (int)k, 0, 32, st));
    } else if (vb == 8) {
        const double *vi = static_cast<const double *>(xv);
        double *vo = c->sort_x_val.as<double>();
        TSMV_CUDA(cub::DeviceRadixSort::SortPairs(nullptr, tb, xi, ko, vi, vo, (int)k, 0, 32, st));
        c->sort_tmp.ensure(tb);
        TSMV_CUDA(cub::DeviceRadixSort::SortPairs(c->sort_tmp.p, tb, xi, ko, vi, vo, (int)k, 0, 32, st));
    } else {
        const float *vi = static_cast<const float *>(xv);
        float *vo = c->sort_x_val.as<float>();
        TSMV_CUDA(cub::DeviceRadixSort::SortPairs(nullptr, tb, xi, ko, vi, vo, (int)k, 0, 32, st));
        c->sort_tmp.ensure(tb);
        TSMV_CUDA(cub::DeviceRadixSort::SortPairs(c->sort_tmp.p, tb, xi, ko, vi, vo, (int)k, 0, 32, st));
    }
    *xi_out = ko;
    *xv_out = xv ? c->sort_x_val.p : nullptr;
}

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
        if (x_nnz == 0 && !has_comm(c)) return TSMV_OK;  // a collective call always takes part
        const bool f32 = c->dtype == TSMV_F32;
        const size_t vb = f32 ? 4 : 8;
        // stage host inputs
        // pinned (mapped) host x is read by the kernel in place (zero copy: phase A
        // reads each entry once, coalesced); pageable host x is staged
        const int32_t *xi = x_idx;
        const void *xv = (sr == TSMV_OR_AND) ? nullptr : x_val;
        // (a collective call hands x to NCCL: device memory only, so it is staged)
        if (!is_device_ptr(xi)) {
            if (const void *d = has_comm(c) ? nullptr : mapped_device_ptr(xi)) {
                xi = static_cast<const int32_t *>(d);
            } else {
                c->stage_x_idx.ensure(x_nnz * 4);
                TSMV_CUDA(cudaMemcpyAsync(c->stage_x_idx.p, xi, x_nnz * 4, cudaMemcpyHostToDevice, st));
                xi = c->stage_x_idx.as<int32_t>();
            }
        }
        if (xv && !is_device_ptr(xv)) {
            if (const void *d = has_comm(c) ? nullptr : mapped_device_ptr(xv)) {
                xv = d;
            } else {
                c->stage_x_val.ensure(x_nnz * vb);
                TSMV_CUDA(cudaMemcpyAsync(c->stage_x_val.p, xv, x_nnz * vb, cudaMemcpyHostToDevice, st));
                xv = c->stage_x_val.p;
            }
        }
        if (has_comm(c)) {
            // distributed: x entries owned by the ranks -> one global ascending x
            x_nnz = comm_gather_x(c, x_nnz, xi, xv, vb, &xi, &xv, st);
            c->last_x_nnz = x_nnz;
            if (x_nnz == 0) return TSMV_OK;
        }
        bool host_y = (y_cap > 0) && !is_device_ptr(y_idx);
        bool host_yv = (y_cap > 0) && sr != TSMV_OR_AND && y_val && !is_device_ptr(y_val);
        int32_t *yi = y_idx;
        void *yv = (sr == TSMV_OR_AND) ? nullptr : y_val;
        int64_t ycap_dev = y_cap;
        // pinned (mapped) host y: copied on the device side (coalesced PCIe writes):
        // by the flat kernel's phase C, each CTA as soon as its pieces are emitted
        // (r2 session 5: 148 -> 142 us end to end at T), else by a copy kernel sized
        // on the device right behind the multiply; then ONE synchronisation for the
        // whole call.  TSMV_Y_DIRECT=1 lets the compaction phase write y into
        // the host buffers itself: measured 1.9x slower end to end at T (its
        // scattered stores cross PCIe one by one; profiles/r02_pb_experiment.txt).
        // Pageable host y is staged on the device and copied after the sync.
        void *myi = host_y ? mapped_device_ptr(y_idx) : nullptr;
        void *myv = host_yv ? mapped_device_ptr(y_val) : nullptr;
        const bool direct = (!host_y || myi) && (!host_yv || myv) && (host_y || host_yv);
        const bool copy_kernel = direct && !getenv("TSMV_Y_DIRECT");
        if (direct && !copy_kernel) {
            if (host_y) yi = static_cast<int32_t *>(myi);
            if (host_yv) yv = myv;
        } else if (host_y || host_yv) {
            ycap_dev = std::min<int64_t>(y_cap, c->m);
            if (host_y) {
                c->stage_y_idx.ensure(std::max<int64_t>(ycap_dev, 1) * 4);
                yi = c->stage_y_idx.as<int32_t>();
            }
            if (host_yv) {
                c->stage_y_val.ensure(std::max<int64_t>(ycap_dev, 1) * vb);
                yv = c->stage_y_val.p;
            }
        }
        volatile Counters *h = c->hcnt;
        int err = 0;
        for (int attempt = 0; attempt < 2; ++attempt) {
            // pinned host y: the flat kernel's phase C copies each CTA's finished rows
            // there itself (TSMV_Y_COPY_KERNEL=1: the separate copy kernel of r2)
            c->hy_by_kernel = false;
            if (copy_kernel && !getenv("TSMV_Y_COPY_KERNEL")) {
                c->hy_idx = host_y ? static_cast<int32_t *>(myi) : nullptr;
                c->hy_val = host_yv ? myv : nullptr;
            }
            enqueue_spmspv(c, sr, x_nnz, xi, xv, ycap_dev, yi, yv, nullptr, st);
            c->hy_idx = nullptr;
            c->hy_val = nullptr;
            if (copy_kernel && !c->hy_by_kernel) {
                k_copy_y<<<c->sm_count * 4, 256, 0, st>>>(yi, yv, &c->counters.as<Counters>()->y_nnz, y_cap,
                                                           static_cast<int32_t *>(myi), myv, (int)vb);
                TSMV_CUDA(cudaGetLastError());
            }
            TSMV_CUDA(cudaStreamSynchronize(st));
            err = h->err;
            if (!err || attempt) break;
            sort_x(c, x_nnz, xi, xv, vb, &xi, &xv, st);  // R21: any order of unique indices
        }
        int64_t ynnz = h->y_nnz;
        TSMV_REQUIRE(err == 0, "tsmv_spmspv: x indices must be unique and in [0, %lld)", (long long)c->n);
        *y_nnz = ynnz;
        if (ynnz > y_cap) {
            set_error("tsmv_spmspv: y_cap %lld < y_nnz %lld", (long long)y_cap, (long long)ynnz);
            return TSMV_ECAPACITY;
        }
        if (!direct) {
            if (host_y) TSMV_CUDA(cudaMemcpyAsync(y_idx, yi, ynnz * 4, cudaMemcpyDeviceToHost, st));
            if (host_yv) TSMV_CUDA(cudaMemcpyAsync(y_val, yv, ynnz * vb, cudaMemcpyDeviceToHost, st));
            if (host_y || host_yv) TSMV_CUDA(cudaStreamSynchronize(st));
        }
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
        TSMV_REQUIRE(!has_comm(c), "tsmv_spmspv_async: a distributed context's call is collective (tsmv_spmspv)");
        TSMV_REQUIRE(is_device_ptr(x_idx) && (sr == TSMV_OR_AND || is_device_ptr(x_val)) &&
                         (y_cap == 0 || is_device_ptr(y_idx)) &&
                         (sr == TSMV_OR_AND || y_cap == 0 || is_device_ptr(y_val)) &&
                         (y_nnz_dev == nullptr || is_device_ptr(y_nnz_dev)),
                     "tsmv_spmspv_async: every pointer must be device memory");
        TSMV_CUDA(cudaSetDevice(c->device));
        c->last_x_nnz = x_nnz;
        enqueue_spmspv(c, sr, x_nnz, x_idx, sr == TSMV_OR_AND ? nullptr : x_val, y_cap, y_idx,
                       sr == TSMV_OR_AND ? nullptr : y_val, (long long *)y_nnz_dev, (cudaStream_t)cuda_stream);
        return TSMV_OK;
    } catch (const Err &e) {
        return e.st;
    }
}

extern "C" int64_t tsmv_trace_words(const tsmv_ctx *c) {
    return c ? (int64_t)c->fused_blocks * (FB / 32) * 8 : 0;
}

extern "C" tsmv_status tsmv_set_trace(tsmv_ctx *c, void *device_buffer) {
    if (!c) return TSMV_EINVAL;
    c->trace = device_buffer;
    return TSMV_OK;
}

extern "C" tsmv_status tsmv_set_direction_rule(tsmv_ctx *c, double push_csr_density, double pull_alpha,
                                               int32_t force_dir) {
    try {
        TSMV_REQUIRE(c, "tsmv_set_direction_rule: NULL ctx");
        TSMV_REQUIRE(push_csr_density > 0 && pull_alpha > 0, "tsmv_set_direction_rule: thresholds must be > 0");
        TSMV_REQUIRE(force_dir >= TSMV_DIR_AUTO && force_dir <= TSMV_DIR_PULL_CSC,
                     "tsmv_set_direction_rule: force_dir out of range");
        c->opt.push_csr_density = push_csr_density;
        c->opt.pull_alpha = pull_alpha;
        c->opt.force_dir = force_dir;
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
