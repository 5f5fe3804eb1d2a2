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
//     64-byte TileRec64 per hit (descriptor + the tile's 16 index bytes inline when
//     nnz <= 16, else its 16 column starts, + its values when they fit), and the
//     useful nonzeros of the warp's other hit tiles are redistributed over the
//     lanes with shuffles (no shared memory);
//   * side work (very sparse tiles, Alg 2 column merge) in 128-item chunks whose
//     list window (start, x_j) is staged in shared memory;
//   * chunks are dealt round-robin to warps (no work-queue atomics on one address);
//   * compaction with one thread per bitmap word (loads of its set rows batched).
// Phases: A | barrier | B1 (a3, a5) -> B2 (a4, own hits, CTA barrier only) | barrier | C write y.
// The touched rows of every bitmap piece are counted at their first touch in B,
// so C needs no counting pass and no barrier of its own (round 2).
#include "spmspv_common.cuh"
#include <algorithm>
#include <cstdlib>
#include <vector>

namespace tsmv {

namespace {

#ifndef TSMV_FT
#define TSMV_FT 1024
#endif
constexpr int FT = TSMV_FT;       // threads per CTA
constexpr int NWF = FT / 32;      // warps per CTA
#ifndef TSMV_TL
#define TSMV_TL 7
#endif
#ifndef TSMV_SL
#define TSMV_SL 7
#endif
constexpr int TL = TSMV_TL;       // log2 tile items per warp task (phase B1)
constexpr int UT = (1 << TL) / 32;
constexpr int SL = TSMV_SL;       // log2 side items per warp chunk
constexpr int US = (1 << SL) / 32;
constexpr int WL = TL > SL ? TL : SL;  // log2 of the per-warp list windows (entries + 1)
#ifndef TSMV_BATCH
#define TSMV_BATCH 4
#endif
#ifndef TSMV_SPW
#define TSMV_SPW 4
#endif
constexpr int SPW = TSMV_SPW;     // set rows up to which a bitmap word is emitted by its own thread
constexpr int BATCH = TSMV_BATCH; // accumulator loads in flight per thread in C2
constexpr int FLAT_TRING = 4096;
constexpr unsigned long long T_CNT_SHIFT = 40, S_CNT_SHIFT = 37;
constexpr long long INF64 = 0x7fffffffffffffffLL;

struct FlatArgs {
    const int32_t *x_idx;
    const void *x_val;
    long long k, n, m, W, row_begin;
    const long long *tptr;
    const uint16_t *mask;
    const TileRec64 *rec;
    const ColInfo *colinfo;
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
    unsigned *pc;       // touched rows per bitmap piece, this call (zero on entry)
    unsigned *pc_next;  // the other buffer: zeroed here for the next call
    int ps_log;         // a piece is 2^ps_log bitmap words
    int n_pieces;
    Counters *cnt;
    Counters *hm;
    unsigned long long bar_base;
    unsigned long long *tring;
    long long tslot;
    const int32_t *hot_list;
    int n_hot;
    unsigned long long *trace;  // tsmv_set_trace: per CTA 8 globaltimer stamps (dev aid)
    int32_t *hy_idx;            // mapped pinned host y of a synchronous call (or null): phase C copies there
    void *hy_val;
    // row buckets (propagation blocking, r2 session 5): products are
    // staged per CTA in shared memory, written to the staging region of their row
    // bucket (2^pb_bl rows) and merged bucket by bucket in shared memory in phase C
    const long long *pb_rs;      // int64[NB + 1]: staging region of bucket q = nonzeros of its rows
    unsigned *pb_row;            // staging: row inside the bucket; phase C output: local row
    unsigned long long *pb_val;  // staging: the product in accumulator encoding
    unsigned *pb_cnt;            // u32[NB]: staged products of bucket q | flags (PB_CNT)
    unsigned *pb_cnt_next;       // the other parity's counters: zeroed here for the next call
    unsigned long long *pb_agg;  // u64[G]: (epoch << 32) | output rows of CTA b (look-back)
    unsigned long long *pb_pu;   // u64[G]: (epoch << 32) | length of CTA b's contributed partial list
    unsigned long long *pb_hp;   // u64[G][n_slots]: hot-row partials of CTA b (EMPTY = untouched)
    unsigned long long *pb_hr;   // u64[n_slots]: reduced hot-row values of this call
    unsigned *pb_hre;            // u32[n_slots]: epoch of pb_hr[slot] (published)
    const int *pb_hs;            // hot slots grouped by bucket: slots of bucket q = pb_hs[pb_hso[q] .. pb_hso[q+1])
    const int *pb_hso;
    unsigned pb_epoch;
    int pb_bl, pb_nb, pb_cap;    // bucket width log2, bucket count, staged products per CTA in shared memory
    long long pb_ovh;            // phase-C weight of a non-empty bucket (its bitmap work), in products
};

// A contribution a*x in accumulator encoding (spmspv_common.cuh): the fp64
// product (-0.0 -> +0.0), the min-second key of x, or nothing (Boolean).
template <int SR> __device__ __forceinline__ unsigned long long enc_prod(double av, double xv) {
    if constexpr (SR == TSMV_PLUS_TIMES) return (unsigned long long)__double_as_longlong(prod_nz(av, xv));
    else if constexpr (SR == TSMV_MIN_SECOND) return ~ord_key(xv) ^ EMPTY;
    else return 0ull;
}
// Combine an encoded partial value into the global accumulator; true if the row
// was untouched (EMPTY) before.
template <int SR> __device__ __forceinline__ bool acc_combine_first(double *acc, long long row, unsigned long long v) {
    if constexpr (SR == TSMV_PLUS_TIMES)
        return (unsigned long long)__double_as_longlong(atomicAdd(&acc[row], __longlong_as_double((long long)v))) == EMPTY;
    else if constexpr (SR == TSMV_MIN_SECOND)
        return (unsigned long long)atomicMax((long long *)&acc[row], (long long)v) == EMPTY;
    else
        return atomicExch((unsigned long long *)&acc[row], 0ull) == EMPTY;
}
// Combine into a shared-memory accumulator slot (several threads: atomics).
template <int SR> __device__ __forceinline__ void sacc_combine(double *s, int r, unsigned long long v) {
    if constexpr (SR == TSMV_PLUS_TIMES) atomicAdd(&s[r], __longlong_as_double((long long)v));
    else if constexpr (SR == TSMV_MIN_SECOND) atomicMax((long long *)&s[r], (long long)v);
}
// The same for a slot owned by the calling thread.
template <int SR> __device__ __forceinline__ void sacc_combine_own(double *s, int r, unsigned long long v) {
    if constexpr (SR == TSMV_PLUS_TIMES) s[r] = s[r] + __longlong_as_double((long long)v);
    else if constexpr (SR == TSMV_MIN_SECOND) {
        const long long o = __double_as_longlong(s[r]);
        if ((long long)v > o) s[r] = __longlong_as_double((long long)v);
    }
}

// Bucket counter: staged products (bits 0-29), a hot row touched (bit 30), rows
// in the global accumulator from a staging-buffer overflow (bit 31).
constexpr unsigned PB_CNT = 0x3fffffffu;

// Per-CTA product staging buffer in shared memory (bucketed variant).
struct PBS {
    unsigned *cur;             // products staged so far by the CTA
    unsigned *row;             // [cap] local row
    unsigned long long *val;   // [cap] encoded value
    int cap;
};
// Stage one product (row >= 0, encoded value v).  Slots are reserved with one
// shared-memory atomic per warp (the lanes that stage together).  Beyond the
// buffer's capacity the product goes to the global accumulator instead; its
// row's touched bit is set and its bucket flagged, and phase C merges it.
template <int SR>
__device__ __forceinline__ void stage(const FlatArgs &a, const PBS &s, long long row, unsigned long long v) {
    const unsigned am = __activemask();
    const int lane = threadIdx.x & 31;
    const int leader = __ffs(am) - 1;
    unsigned base = 0;
    if (lane == leader) base = atomicAdd(s.cur, (unsigned)__popc(am));
    base = __shfl_sync(am, base, leader);
    const unsigned slot = base + (unsigned)__popc(am & ((1u << lane) - 1u));
    if (slot < (unsigned)s.cap) {
        s.row[slot] = (unsigned)row;
        s.val[slot] = v;
        return;
    }
    if (acc_combine_first<SR>(a.acc, row, v)) {
        atomicOr(&a.rowbits[row >> 5], 1u << (row & 31));
        atomicOr(&a.pb_cnt[row >> a.pb_bl], 0x80000000u);
    }
}

// One contribution a*x to row code `rc` (>= 0: local row; < 0: ~hot slot).
// Returns the row whose touched bit must be set (first contribution), or -1.
// Bucketed variant (PB): the product is staged and -1 returned.
template <int SR, bool PB>
__device__ __forceinline__ long long contribute(const FlatArgs &a, double *s_hacc, uint32_t *s_hbits, const PBS &ps,
                                                long long rc, double av, double xv) {
    if (rc < 0) {
        const int sl = (int)~rc;
        acc_shared<SR>(s_hacc, sl, av, xv);
        atomicOr(&s_hbits[sl >> 5], 1u << (sl & 31));
        return -1;
    }
    if constexpr (PB) {
        stage<SR>(a, ps, rc, enc_prod<SR>(av, xv));
        return -1;
    } else {
        return acc_first<SR>(a.acc, rc, av, xv) ? rc : -1;
    }
}
// first touch of `row` (>= 0; -1 = none): its bit, and its piece's count in the
// CTA's shared-memory counters (added to the global ones once, at the end of B)
__device__ __forceinline__ void touch(const FlatArgs &a, unsigned *s_pc, long long row) {
    if (row >= 0) {
        atomicOr(&a.rowbits[row >> 5], 1u << (row & 31));
        atomicAdd(&s_pc[(row >> 5) >> a.ps_log], 1u);
    }
}


constexpr int HEAVY_CAP = 128;
constexpr int MAXG = 256;  // max CTAs of the flat kernel (one per SM)
constexpr int KP = 8;      // bitmap pieces per CTA in phase C
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

__device__ __forceinline__ ColInfo load_colinfo(const ColInfo *p) {
    const longlong2 v = __ldg(reinterpret_cast<const longlong2 *>(p));
    ColInfo c;
    c.sbeg = v.x;
    c.tinfo = (unsigned long long)v.y;
    return c;
}

__device__ __forceinline__ unsigned ld_acquire_u32(const unsigned *p) {
    unsigned v;
    asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ unsigned ld_relaxed_u32(const unsigned *p) {
    unsigned v;
    asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ unsigned long long ld_relaxed_u64(const unsigned long long *p) {
    unsigned long long v;
    asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_release_u32(unsigned *p, unsigned v) {
    asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ void st_release_u64(unsigned long long *p, unsigned long long v) {
    asm volatile("st.release.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}

// Bucketed variant, end of phase B.  The CTA's privatised hot-row partials go
// to its row of pb_hp (coalesced, EMPTY where untouched; phase C reduces them
// over the CTAs).  The staged products are counting-sorted by bucket in shared
// memory (rank per product, bucket starts by a block scan, permutation), one
// global reservation per (CTA, non-empty bucket) places the CTA's run in the
// bucket's staging region, and the sorted products are stored with consecutive
// threads writing consecutive positions of each run.
template <int SR>
__device__ void pb_flush(const FlatArgs &a, const PBS &ps, const double *s_hacc, const uint32_t *s_hbits,
                         int n_slots, unsigned *s_bhist, long long *s_bbase, unsigned short *s_brank,
                         unsigned short *s_perm, bool err, long long (*s_acct)[4], long long (*s_scan)[NWF],
                         unsigned long long *tr) {
    const int tid = threadIdx.x, b = blockIdx.x;
    if (tid < 4) {
        long long sum = 0;
        for (int w = 0; w < NWF; ++w) sum += s_acct[w][tid];
        a.acct[b * 4 + tid] = sum;
    }
    if (err) return;
    const int BL = a.pb_bl, NB = a.pb_nb;
    for (int q = tid; q < n_slots; q += FT) {
        const bool t = (s_hbits[q >> 5] >> (q & 31)) & 1u;
        a.pb_hp[(long long)b * n_slots + q] =
            !t ? EMPTY : (SR == TSMV_OR_AND ? 0ull : (unsigned long long)__double_as_longlong(s_hacc[q]));
    }
    if (tr && tid == 0) tr[12] = globaltimer_ns();
    const int nb = (int)min(*ps.cur, (unsigned)ps.cap);
    for (int i = tid; i < nb; i += FT) s_brank[i] = (unsigned short)atomicAdd(&s_bhist[ps.row[i] >> BL], 1u);
    __syncthreads();
    if (tr && tid == 0) tr[13] = globaltimer_ns();
    {
        constexpr int PPT = 4;  // NB <= 4 * FT (host)
        long long h[PPT], run = 0;
#pragma unroll
        for (int i = 0; i < PPT; ++i) {
            const int q = tid * PPT + i;
            h[i] = q < NB ? (long long)s_bhist[q] : 0;
            run += h[i];
        }
        long long ex, tot;
        block_scan<1, FT>(&run, &ex, &tot, s_scan);
#pragma unroll
        for (int i = 0; i < PPT; ++i) {
            const int q = tid * PPT + i;
            if (q < NB) {
                s_bhist[q] = (unsigned)ex;  // now the bucket's first sorted slot
                if (h[i])
                    s_bbase[q] = __ldg(&a.pb_rs[q]) + (long long)(atomicAdd(&a.pb_cnt[q], (unsigned)h[i]) & PB_CNT) - ex;
            }
            ex += h[i];
        }
    }
    __syncthreads();
    if (tr && tid == 0) tr[14] = globaltimer_ns();
    for (int i = tid; i < nb; i += FT) s_perm[s_bhist[ps.row[i] >> BL] + s_brank[i]] = (unsigned short)i;
    __syncthreads();
    const unsigned lm = (1u << BL) - 1u;
    for (int j = tid; j < nb; j += FT) {
        const int i = s_perm[j];
        const unsigned r = ps.row[i];
        const long long pos = s_bbase[r >> BL] + j;
        a.pb_row[pos] = r & lm;
        a.pb_val[pos] = ps.val[i];
    }
}

// CTA of weight position `pos`: the largest c with floor(W c / G) <= pos.
__device__ __forceinline__ int pb_cta_of(long long pos, long long W, int G) {
    int lo = 0, hi = G - 1;
    while (lo < hi) {
        const int mid = (lo + hi + 1) >> 1;
        if (W * mid / G <= pos) lo = mid;
        else hi = mid - 1;
    }
    return lo;
}

// Semiring join of two encoded partial values (EMPTY is the identity).
template <int SR> __device__ __forceinline__ unsigned long long pb_join(unsigned long long x, unsigned long long y) {
    if constexpr (SR == TSMV_PLUS_TIMES)
        return (unsigned long long)__double_as_longlong(__longlong_as_double((long long)x) +
                                                       __longlong_as_double((long long)y));
    else if constexpr (SR == TSMV_MIN_SECOND)
        return (long long)x > (long long)y ? x : y;
    else
        return (x == EMPTY && y == EMPTY) ? EMPTY : 0ull;
}

// Accumulate a list of (row inside the bucket, encoded value) pairs into the
// CTA's shared-memory bucket (UN loads in flight per thread).
template <int SR>
__device__ __forceinline__ void pb_accumulate(const unsigned *rows, const unsigned long long *vals, long long n,
                                              double *c_acc, unsigned *c_bits) {
    constexpr int UN = 4;
    const int tid = threadIdx.x;
    for (long long i0 = 0; i0 < n; i0 += (long long)UN * FT) {
        unsigned r[UN];
        unsigned long long v[UN];
#pragma unroll
        for (int u = 0; u < UN; ++u) {
            const long long i = i0 + tid + (long long)u * FT;
            r[u] = 0xffffffffu;
            if (i < n) {
                r[u] = __ldcg(&rows[i]);
                v[u] = __ldcg(&vals[i]);
            }
        }
#pragma unroll
        for (int u = 0; u < UN; ++u) {
            if (r[u] != 0xffffffffu) {
                sacc_combine<SR>(c_acc, (int)r[u], v[u]);
                atomicOr(&c_bits[r[u] >> 5], 1u << (r[u] & 31));
            }
        }
    }
}

// Write the CTA's shared-memory bucket as a compact list (rows ascending, row
// code = row0 + row inside the bucket) and clear it; returns the list length
// (all threads).
__device__ __forceinline__ long long pb_compact(double *c_acc, unsigned *c_bits, unsigned *c_wex, int WB,
                                                long long (*s_scan)[NWF], unsigned *dst_row,
                                                unsigned long long *dst_val, long long row0) {
    const int tid = threadIdx.x, NWB = WB >> 5;
    long long pc = tid < NWB ? __popc(c_bits[tid]) : 0, wex, ub;
    block_scan<1, FT>(&pc, &wex, &ub, s_scan);
    if (tid < NWB) c_wex[tid] = (unsigned)wex;
    __syncthreads();
    for (int r = tid; r < WB; r += FT) {
        const unsigned wb = c_bits[r >> 5];
        if ((wb >> (r & 31)) & 1u) {
            const long long pos = c_wex[r >> 5] + __popc(wb & ((1u << (r & 31)) - 1u));
            dst_row[pos] = (unsigned)(row0 + r);
            dst_val[pos] = (unsigned long long)__double_as_longlong(c_acc[r]);
            c_acc[r] = __longlong_as_double((long long)EMPTY);
        }
    }
    __syncthreads();
    if (tid < NWB) c_bits[tid] = 0u;
    return ub;
}

// Bucketed variant, phase C (a6).  Bucket q weighs its staged products plus
// pb_ovh (if non-empty); the weight line is cut into G equal ranges and CTA b
// takes the products in its range.  A bucket wholly inside one range is merged
// by that CTA alone in shared memory (dense 2^BL-row accumulator + bitmap).  A
// bucket spanning several ranges is "shared": each CTA after its first one
// (a contributor; a CTA contributes to at most one bucket, its first) merges
// its share, writes it back compacted in place over that share and publishes
// the length (pb_pu[c], epoch-tagged); the first CTA (the emitter) merges its
// own share and the contributors' lists.  Rows in the global accumulator (hot
// rows, staging-buffer overflow: the bucket's bit 31) are merged by the emitter
// from the touched bitmap.  Every CTA compacts its emitted buckets, in bucket
// order, into the staging region from its first emitted bucket on (in place: a
// bucket has at most as many output rows as nonzeros), then finds its y offset
// by look-back over the CTAs before it and copies its rows to y.
template <int SR, class XV>
__device__ void pb_emit(const FlatArgs &a, bool err, long long (*s_scan)[NWF], unsigned char *s_dyn,
                        int n_slots, unsigned long long *tr) {
    __shared__ int s_qlo, s_qhi;
    __shared__ long long s_off, s_u, s_pl;
    const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
    const int G = gridDim.x, b = blockIdx.x;
    const int BL = a.pb_bl, NB = a.pb_nb;
    const int WB = 1 << BL, NWB = WB >> 5;
    double *c_acc = reinterpret_cast<double *>(s_dyn);             // [WB]
    unsigned *c_bits = reinterpret_cast<unsigned *>(c_acc + WB);    // [NWB]
    unsigned *c_wex = c_bits + NWB;                                 // [NWB]
    long long *s_S = reinterpret_cast<long long *>(c_wex + NWB);    // [NB]: weight prefix of bucket q
    long long U = 0, out0 = -1;
    if (!err) {
        for (int i = tid; i < WB; i += FT) c_acc[i] = __longlong_as_double((long long)EMPTY);
        for (int i = tid; i < NWB; i += FT) c_bits[i] = 0u;
        constexpr int PPT = 4;  // NB <= 4 * FT (host)
        long long wv[PPT], run = 0;
#pragma unroll
        for (int i = 0; i < PPT; ++i) {
            const int q = tid * PPT + i;
            wv[i] = 0;
            if (q < NB) {
                const unsigned cv = __ldcg(&a.pb_cnt[q]);
                const long long c = cv & PB_CNT;
                const bool hot = n_slots && __ldg(&a.pb_hso[q + 1]) > __ldg(&a.pb_hso[q]);
                wv[i] = (cv || hot) ? c + a.pb_ovh : 0;
            }
            run += wv[i];
        }
        long long ex, Wt;
        block_scan<1, FT>(&run, &ex, &Wt, s_scan);
        const long long lo = Wt * b / G, hi = Wt * (b + 1) / G;
        if (tid == 0) {
            s_qlo = NB;
            s_qhi = -1;
        }
        __syncthreads();
#pragma unroll
        for (int i = 0; i < PPT; ++i) {
            const int q = tid * PPT + i;
            if (q < NB) {
                s_S[q] = ex;
                if (wv[i] > 0 && ex < hi && ex + wv[i] > lo) {
                    atomicMin(&s_qlo, q);
                    atomicMax(&s_qhi, q);
                }
            }
            ex += wv[i];
        }
        __syncthreads();
        // hot rows: warp w of the grid reduces the CTAs' partials of hot slot w and
        // publishes the result (epoch-tagged) for the bucket's emitter
        for (int sl = b * NWF + wid; sl < n_slots; sl += G * NWF) {
            constexpr int NP = MAXG / 32;
            unsigned long long v[NP];
#pragma unroll
            for (int i = 0; i < NP; ++i)
                v[i] = lane + 32 * i < G ? __ldcg(&a.pb_hp[(long long)(lane + 32 * i) * n_slots + sl]) : EMPTY;
            unsigned long long t = EMPTY;
#pragma unroll
            for (int i = 0; i < NP; ++i) t = pb_join<SR>(t, v[i]);
#pragma unroll
            for (int o = 16; o > 0; o >>= 1) t = pb_join<SR>(t, __shfl_xor_sync(0xffffffffu, t, o));
            if (lane == 0) {
                a.pb_hr[sl] = t;
                st_release_u32(&a.pb_hre[sl], a.pb_epoch);
            }
        }
        const int q0 = s_qlo, q1 = s_qhi;
        if (tr && tid == 0) tr[15] = (unsigned long long)(q1 - q0 + 1) * 1000ull;  // dev aid: buckets met (x1000 for the us print)
        for (int q = q0; q <= q1; ++q) {
            const unsigned cv = __ldcg(&a.pb_cnt[q]);
            const long long cq = cv & PB_CNT;
            const bool ovf = (cv >> 31) != 0u;
            const int h0 = n_slots ? __ldg(&a.pb_hso[q]) : 0, h1 = n_slots ? __ldg(&a.pb_hso[q + 1]) : 0;
            if (!cv && h1 == h0) continue;
            const long long Sq = s_S[q];
            const long long p0 = max(lo, Sq) - Sq, p1 = min(hi, Sq + cq) - Sq;
            const bool emit = Sq >= lo && Sq < hi;
            if (!emit && p1 <= p0) continue;
            const long long rs = __ldg(&a.pb_rs[q]);
            if (p1 > p0) pb_accumulate<SR>(a.pb_row + rs + p0, a.pb_val + rs + p0, p1 - p0, c_acc, c_bits);
            const long long grow0 = (long long)q << BL;
            if (emit) {
                // hot rows of the bucket: the reduced partials published above
                for (int h = h0 + tid; h < h1; h += FT) {
                    const int sl = __ldg(&a.pb_hs[h]);
                    while (ld_relaxed_u32(&a.pb_hre[sl]) != a.pb_epoch) {
                    }
                    (void)ld_acquire_u32(&a.pb_hre[sl]);
                    const unsigned long long t = __ldcg(&a.pb_hr[sl]);
                    if (t != EMPTY) {
                        const long long row = (long long)__ldg(&a.hot_list[sl / 16]) * 16 + sl % 16;
                        const int r = (int)(row - grow0);
                        sacc_combine<SR>(c_acc, r, t);
                        atomicOr(&c_bits[r >> 5], 1u << (r & 31));
                    }
                }
            }
            __syncthreads();
            if (!emit) {
                // a later share of a shared bucket: compacted in place, length published
                const long long u = pb_compact(c_acc, c_bits, c_wex, WB, s_scan, a.pb_row + rs + p0,
                                               a.pb_val + rs + p0, 0);
                __threadfence();
                __syncthreads();
                if (tid == 0)
                    st_release_u64(&a.pb_pu[b], ((unsigned long long)a.pb_epoch << 32) | (unsigned long long)u);
                continue;
            }
            if (cq > 0 && p1 < cq) {
                // the contributors: the CTAs after b whose (non-empty) range meets the
                // bucket (every range is non-empty once Wt >= G)
                const int last = pb_cta_of(Sq + cq - 1, Wt, G);
                for (int c = b + 1; c <= last; ++c) {
                    const long long loc = Wt * c / G;
                    if (loc >= Wt * (c + 1) / G) continue;
                    if (tid == 0) {
                        unsigned long long v;
                        do {
                            v = ld_acquire_u64(&a.pb_pu[c]);
                        } while ((unsigned)(v >> 32) != a.pb_epoch);
                        s_pl = (long long)(v & 0xffffffffull);
                    }
                    __syncthreads();
                    const long long off = rs + (loc - Sq);
                    pb_accumulate<SR>(a.pb_row + off, a.pb_val + off, s_pl, c_acc, c_bits);
                    __syncthreads();
                }
            }
            if (ovf) {
                // the bucket's rows in the global accumulator (clear on read); 4 rows
                // per thread in flight
                const int IT = WB / FT;
                for (int i0 = 0; i0 < IT; i0 += 4) {
                    unsigned wb[4];
                    unsigned long long v[4];
#pragma unroll
                    for (int u = 0; u < 4; ++u) {
                        const long long row = grow0 + tid + (long long)(i0 + u) * FT;
                        wb[u] = (i0 + u < IT && row < a.m) ? __ldcg(&a.rowbits[row >> 5]) : 0u;
                    }
#pragma unroll
                    for (int u = 0; u < 4; ++u) {
                        const long long row = grow0 + tid + (long long)(i0 + u) * FT;
                        if ((wb[u] >> lane) & 1u) v[u] = (unsigned long long)__ldcg((const long long *)&a.acc[row]);
                    }
#pragma unroll
                    for (int u = 0; u < 4; ++u) {
                        const int r = tid + (i0 + u) * FT;
                        const bool set = (wb[u] >> lane) & 1u;
                        if (set) {
                            a.acc[grow0 + r] = __longlong_as_double((long long)EMPTY);
                            sacc_combine_own<SR>(c_acc, r, v[u]);
                        }
                        const unsigned bal = __ballot_sync(0xffffffffu, set);
                        if (lane == 0 && bal) {
                            c_bits[r >> 5] |= bal;
                            a.rowbits[(grow0 + r) >> 5] = 0u;
                        }
                    }
                }
                __syncthreads();
            }
            if (out0 < 0) out0 = rs;
            U += pb_compact(c_acc, c_bits, c_wex, WB, s_scan, a.pb_row + out0 + U, a.pb_val + out0 + U, grow0);
            __syncthreads();
        }
    }
    // look-back: y offset of this CTA = output rows of the CTAs before it
    if (tid == 0) st_release_u64(&a.pb_agg[b], ((unsigned long long)a.pb_epoch << 32) | (unsigned long long)U);
    if (tr && tid == 0) tr[10] = globaltimer_ns();
    if (wid == 0) {
        // all predecessors' aggregates polled at once (relaxed: only the counts are used)
        constexpr int NP = MAXG / 32;
        unsigned long long v[NP];
        const unsigned long long ready = (unsigned long long)a.pb_epoch << 32;
#pragma unroll
        for (int i = 0; i < NP; ++i) v[i] = lane + 32 * i < b ? ld_relaxed_u64(&a.pb_agg[lane + 32 * i]) : ready;
        long long s = 0;
#pragma unroll
        for (int i = 0; i < NP; ++i) {
            while ((unsigned)(v[i] >> 32) != a.pb_epoch) v[i] = ld_relaxed_u64(&a.pb_agg[lane + 32 * i]);
            s += (long long)(v[i] & 0xffffffffull);
        }
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
        if (lane == 0) {
            s_off = s;
            s_u = U;
        }
    }
    __syncthreads();
    if (tr && tid == 0) tr[11] = globaltimer_ns();
    const long long off = s_off;
    for (long long i = tid; i < U; i += FT) {
        const long long pos = off + i;
        if (pos < a.y_cap) {
            const unsigned row = __ldcg(&a.pb_row[out0 + i]);
            a.y_idx[pos] = (int32_t)((long long)row + a.row_begin);
            if (a.y_val) {
                const unsigned long long v = __ldcg(&a.pb_val[out0 + i]);
                double x = __longlong_as_double((long long)v);
                if constexpr (SR == TSMV_MIN_SECOND) x = ord_val(~(v ^ EMPTY));
                ((XV *)a.y_val)[pos] = (XV)x;
            }
        }
    }
    if (b == G - 1 && tid == 0) {
        const long long yt = off + U;
        a.cnt->y_nnz = yt;
        a.hm->y_nnz = yt;
        if (a.ynnz_dev) *a.ynnz_dev = err ? -1 : yt;
    }
}

// dynamic shared memory of phase B before the bucketed variant's staging buffer
constexpr size_t FLAT_DYN_B0 = HOT_SLOTS * 8 + (size_t)NWF * ((1 << WL) + 1) * 24 + HOT_SLOTS / 8;
constexpr size_t pb_align(size_t x) { return (x + 15) & ~(size_t)15; }

template <class AV, class XV, int SR, bool PB>
__global__ void __launch_bounds__(FT, 1) k_spmspv_flat(FlatArgs a) {
    constexpr int NT = 16, LOG = 4;
    constexpr int WN = (1 << WL) + 1;
    __shared__ long long s_scan[8][NWF];
    extern __shared__ __align__(16) unsigned char s_dyn[];
    double *s_hacc = reinterpret_cast<double *>(s_dyn);                           // [HOT_SLOTS]
    long long *s_win = reinterpret_cast<long long *>(s_dyn + HOT_SLOTS * 8);      // [NWF][WN]
    long long *s_winb = s_win + NWF * WN;                                         // [NWF][WN]
    double *s_winx = reinterpret_cast<double *>(s_winb + NWF * WN);               // [NWF][WN]
    uint32_t *s_hbits = reinterpret_cast<uint32_t *>(s_winx + NWF * WN);          // [HOT_SLOTS/32]
    unsigned *s_pcnt = s_hbits + HOT_SLOTS / 32;                                  // [MAXG * KP] (flat)
    // bucketed variant: per-bucket base i64[NB], staged values u64[cap], per-bucket
    // counts u32[NB], staged rows u32[cap], ranks u16[cap], permutation u16[cap]
    // (after s_hbits)
    __shared__ unsigned s_bcur;
    PBS ps;
    long long *s_bbase = nullptr;
    unsigned *s_bhist = nullptr;
    unsigned short *s_brank = nullptr, *s_perm = nullptr;
    if constexpr (PB) {
        const size_t o0 = pb_align(FLAT_DYN_B0);
        s_bbase = reinterpret_cast<long long *>(s_dyn + o0);
        ps.val = reinterpret_cast<unsigned long long *>(s_bbase + a.pb_nb);
        s_bhist = reinterpret_cast<unsigned *>(ps.val + a.pb_cap);
        ps.row = s_bhist + a.pb_nb;
        s_brank = reinterpret_cast<unsigned short *>(ps.row + a.pb_cap);
        s_perm = s_brank + a.pb_cap;
        ps.cur = &s_bcur;
        ps.cap = a.pb_cap;
    } else {
        ps.cur = nullptr;
        ps.row = nullptr;
        ps.val = nullptr;
        ps.cap = 0;
    }
    __shared__ long long s_base[4], s_tot[4];
    __shared__ long long s_acct[NWF][4];
    __shared__ int s_err;
    __shared__ int s_nheavy;
    __shared__ int s_hcnt;
    __shared__ long long s_pbase[KP], s_ex0[KP];
    __shared__ int s_nd;  // dense bitmap words of the current C2 round
    __shared__ int s_hlist[HOT_SLOTS / 16];  // tile rows of the privatised hot rows
    __shared__ long long s_heavy[HEAVY_CAP][3];  // chunk-map runs too long for one thread: c0, c1, list | kind
    const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
    const int G = gridDim.x, b = blockIdx.x;
    unsigned long long target = a.bar_base;
    const bool stamp = a.tring && b == 0 && tid == 0;
    unsigned long long *ts = a.tring ? a.tring + (a.tslot % FLAT_TRING) * 8 : nullptr;
    if (stamp) ts[0] = globaltimer_ns();
    unsigned long long *tr = a.trace ? a.trace + (long long)b * 16 : nullptr;
    if (tr && tid == 0) tr[0] = globaltimer_ns();
    const int n_slots = a.n_hot * NT;
    for (int i = tid; i < n_slots; i += FT) s_hacc[i] = __longlong_as_double((long long)EMPTY);
    for (int i = tid; i < (n_slots + 31) / 32; i += FT) s_hbits[i] = 0u;
    for (int i = tid; i < a.n_hot; i += FT) s_hlist[i] = a.hot_list[i];
    if (tid == 0) {
        s_nheavy = 0;
        s_hcnt = 0;
    }
    if constexpr (PB) {
        for (int i = tid; i < a.pb_nb; i += FT) s_bhist[i] = 0u;
        if (tid == 0) s_bcur = 0u;
        // the next call's bucket counters (this call's were zeroed by the previous one)
        for (long long i = (long long)b * FT + tid; i < a.pb_nb; i += (long long)G * FT) {
            a.pb_cnt_next[i] = 0u;
        }
    } else {
        for (int i = tid; i < a.n_pieces; i += FT) s_pcnt[i] = 0u;
        if (tid < KP && b + tid * G < a.n_pieces) a.pc_next[b + tid * G] = 0u;
    }

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
        const ColInfo ci = load_colinfo(a.colinfo + j);
        const long long ws = __ldg(&a.colinfo[j + 1].sbeg) - ci.sbeg;
        if (e == 0 || (prev >> LOG) != J) {
            const long long wt = (long long)(ci.tinfo & 0xffffffull);
            q[0] += wt > 0;
            q[1] += wt;
        }
        q[2] += ws > 0;
        q[3] += ws;
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
        if (tr) tr[8] = globaltimer_ns();
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
            const ColInfo ci = load_colinfo(a.colinfo + j);
            if (e == 0 || (prev >> LOG) != J) {
                const long long tb = (long long)(ci.tinfo >> 24), wt = (long long)(ci.tinfo & 0xffffffull);
                if (wt > 0) {
                    // the segment's x bits and values (x stored by segment)
                    unsigned mk = 0;
                    double *xs = a.L.t_xv + oLt * NT;
                    for (long long e2 = e; e2 < a.k; ++e2) {
                        const long long j2 = a.x_idx[e2];
                        if ((j2 >> LOG) != J) break;
                        mk |= 1u << (j2 & (NT - 1));
                        xs[j2 & (NT - 1)] = a.x_val ? (double)((const XV *)a.x_val)[e2] : 1.0;
                    }
                    a.L.t_beg[oLt] = tb;
                    a.L.t_wpre[oLt] = oWt;
                    a.L.t_xm[oLt] = mk;
                    put_chunks<TL>(a.L.Ct, oWt, wt, (int)oLt, 0, s_heavy, &s_nheavy);
                    ++oLt;
                    oWt += wt;
                }
            }
            const long long sb = ci.sbeg, ws = __ldg(&a.colinfo[j + 1].sbeg) - sb;
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
    // hit-list region per CTA: the CTA's tile tasks (<= ceil(nTT / G)) x 128 items
    const long long RC = (((s_tot[1] + (1 << TL) - 1) >> TL) + G - 1) / G * (1 << TL);

    // ------------------------------------------------------------ phase B1 (a3, a5)
    // Warp tasks of 128 items, dealt round-robin: a tile task ANDs the column masks
    // of 128 tiles with their segment's x bits (4 mask loads in flight per lane) and
    // appends the hits to a global hit list (one reservation per CTA and round); a
    // side task multiplies 128 side nonzeros (Alg 2 column merge) into acc.
    long long n_hit = 0, n_hcol = 0, n_mac = 0, n_ind = 0;
    const long long nwarps = (long long)G * NWF;
    if (!err) {
        const long long nLt = s_tot[0], Wt = s_tot[1], nLs = s_tot[2], Ws = s_tot[3];
        const long long nTT = (Wt + (1 << TL) - 1) >> TL, nCs = (Ws + (1 << SL) - 1) >> SL;
        const long long ntask = nTT + nCs;
        const long long rounds = (ntask + nwarps - 1) / nwarps;
        (void)rounds;
        const AV *sval = (const AV *)a.sval;
        long long *win = s_win + wid * WN;
        long long *winb = s_winb + wid * WN;
        double *winx = s_winx + wid * WN;
        long long *winp = reinterpret_cast<long long *>(winx);
        for (long long task = (long long)wid * G + b; task < ntask; task += nwarps) {
            unsigned hv[UT];
            long long tv[UT];
            int Jv[UT];
#pragma unroll
            for (int u = 0; u < UT; ++u) hv[u] = 0u;
            if (task < nTT) {
                const long long base = task << TL;
                const long long s0 = __ldcg(&a.L.Ct[task]);
#pragma unroll
                for (int q0 = 0; q0 <= (1 << TL); q0 += 32) {
                    const int qx = q0 + lane;
                    const long long ix = s0 + qx;
                    const bool in = ix < nLt;
                    const long long w = in ? __ldcg(&a.L.t_wpre[ix]) : INF64;
                    const long long tb = in ? __ldcg(&a.L.t_beg[ix]) : 0;
                    const long long pk = in ? (long long)__ldcg(&a.L.t_xm[ix]) : 0;
                    if (qx <= (1 << TL)) {
                        win[qx] = w;
                        winb[qx] = tb;
                        winp[qx] = pk;
                    }
                }
                __syncwarp();
                ChunkMap<TL> cm;
                cm.build(win, base, lane);
                unsigned xm[UT];
#pragma unroll
                for (int u = 0; u < UT; ++u) {
                    const long long i = base + lane + 32 * u;
                    const bool ok = i < Wt;
                    const int qq = ok ? cm.entry(lane + 32 * u) : 0;
                    tv[u] = winb[qq] + (i - win[qq]);
                    const long long pk = winp[qq];
                    xm[u] = ok ? (unsigned)(pk & 0xffff) : 0u;
                    Jv[u] = (int)(s0 + qq);  // list slot of the segment
                }
#pragma unroll
                for (int u = 0; u < UT; ++u) hv[u] = xm[u] ? ((unsigned)__ldg(&a.mask[tv[u]]) & xm[u]) : 0u;
                __syncwarp();
            } else if (task < ntask) {
                const long long c2 = task - nTT;
                const long long base = c2 << SL;
                const long long s0 = __ldcg(&a.L.Cs[c2]);
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
                long long fr[US];
#pragma unroll
                for (int u = 0; u < US; ++u)
                    fr[u] = ok[u] ? contribute<SR, PB>(a, s_hacc, s_hbits, ps, (long long)row[u], av[u], xv[u]) : -1;
#pragma unroll
                for (int u = 0; u < US; ++u) touch(a, s_pcnt, fr[u]);
                __syncwarp();
            }
            // append this round's hits: warp offsets in shared memory, one global
            // reservation per CTA
            int nmine = 0;
#pragma unroll
            for (int u = 0; u < UT; ++u) nmine += hv[u] != 0u;
            int incl = nmine;
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                const int v = __shfl_up_sync(0xffffffffu, incl, o);
                if (lane >= o) incl += v;
            }
            const int wtot = __shfl_sync(0xffffffffu, incl, 31);
            int woff = 0;
            if (lane == 0 && wtot) woff = atomicAdd(&s_hcnt, wtot);
            woff = __shfl_sync(0xffffffffu, woff, 0);
            long long o = (long long)b * RC + woff + incl - nmine;
#pragma unroll
            for (int u = 0; u < UT; ++u)
                if (hv[u]) a.L.hits[o++] = make_uint4((unsigned)tv[u], hv[u], (unsigned)Jv[u], 0u);
        }
    }
    // B2 takes the hits of this CTA only: its list region is complete after this
    // __syncthreads, so there is no grid barrier between B1 and B2 (a CTA whose
    // B1 ends early starts multiplying at once)
    __syncthreads();
    if (tr && tid == 0) tr[3] = globaltimer_ns();
    if (stamp) ts[6] = globaltimer_ns();

    // ------------------------------------------------------------ phase B2 (a4)
    // lane = hit tile: one 64-byte record.  Tiles whose values are inline (and
    // indices, nnz <= 16) are multiplied by their own lane; the useful nonzeros of
    // the other hit tiles of the warp are redistributed over the lanes (shuffles)
    // and read from the idx / val arrays.
    if (!err) {
        const long long NH = s_hcnt;
        const AV *val = (const AV *)a.val;
        constexpr int INL = 32 / (int)sizeof(AV);
        for (long long hb = (long long)wid * 32; hb < NH; hb += NWF * 32) {
            const long long h = hb + lane;
            unsigned hit = 0u;
            long long t = 0;
            int slot = 0;
            double xv0 = 0.0;
            if (h < NH) {
                const uint4 e = __ldcg(&a.L.hits[(long long)b * RC + h]);
                t = e.x;
                hit = e.y;
                slot = (int)e.z;
                // x value of the first hit column, fetched beside the tile record
                xv0 = __ldcg(&a.L.t_xv[(long long)slot * NT + (__ffs(hit) - 1)]);
            }
            unsigned off = 0, nnz = 0;
            int trow = 0;
            uint4 bb = make_uint4(0, 0, 0, 0);
            int useful = 0;
            if (hit) {
                const uint4 *rp = reinterpret_cast<const uint4 *>(a.rec + t);
                uint4 h0, h1, v0, v1;
                ld32_nc(rp, h0, h1);
                ld32_nc(rp + 2, v0, v1);
                off = h0.x;
                trow = (int)h0.y;
                nnz = h0.z;
                bb = h1;
                ++n_hit;
                n_hcol += __popc(hit);
                if (nnz <= (val ? (unsigned)INL : 16u)) {
                    // inline tile: this lane multiplies its useful nonzeros, issuing the
                    // atomics of up to 4 of them before waiting for any "first" result
                    const double *xs = a.L.t_xv + (long long)slot * NT;
                    const int c0 = __ffs(hit) - 1;
                    for (int g = 0; g < (int)nnz; g += 4) {
                        long long fr[4];
#pragma unroll
                        for (int j = 0; j < 4; ++j) {
                            const int p = g + j;
                            fr[j] = -1;
                            const int by = p < (int)nnz ? byte_of(bb, p) : 0xff;
                            const int c = by >> 4, rr = by & (NT - 1);
                            if (p < (int)nnz && ((hit >> c) & 1u)) {
                                double av = 1.0;
                                if (val) {
                                    if constexpr (sizeof(AV) == 8) {
                                        const uint4 &vq = p < 2 ? v0 : v1;
                                        av = (p & 1) ? __hiloint2double((int)vq.w, (int)vq.z)
                                                     : __hiloint2double((int)vq.y, (int)vq.x);
                                    } else {
                                        const uint4 &vq = p < 4 ? v0 : v1;
                                        const int q4 = p & 3;
                                        av = (double)__uint_as_float(q4 == 0 ? vq.x : q4 == 1 ? vq.y : q4 == 2 ? vq.z : vq.w);
                                    }
                                }
                                const double xv = c == c0 ? xv0 : __ldcg(&xs[c]);
                                const long long rc =
                                    trow >= 0 ? (long long)trow * NT + rr : ~((long long)(~trow) * NT + rr);
                                fr[j] = contribute<SR, PB>(a, s_hacc, s_hbits, ps, rc, av, xv);
                                ++n_mac;
                            }
                        }
#pragma unroll
                        for (int j = 0; j < 4; ++j) touch(a, s_pcnt, fr[j]);
                    }
                } else {
                    useful = rec_useful(bb, hit, (int)nnz);
                }
            }
            int incl = useful;
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                const int v = __shfl_up_sync(0xffffffffu, incl, o);
                if (lane >= o) incl += v;
            }
            const int total = __shfl_sync(0xffffffffu, incl, 31);
            n_mac += useful;
            n_ind += useful;
            long long frp = -1, frq = -1;
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
                const unsigned offs = __shfl_sync(0xffffffffu, off, lo);
                const int trs = __shfl_sync(0xffffffffu, trow, lo);
                const int nns = __shfl_sync(0xffffffffu, (int)nnz, lo);
                const unsigned hs = __shfl_sync(0xffffffffu, hit, lo);
                const int ss = __shfl_sync(0xffffffffu, slot, lo);
                uint4 bs;
                bs.x = __shfl_sync(0xffffffffu, bb.x, lo);
                bs.y = __shfl_sync(0xffffffffu, bb.y, lo);
                bs.z = __shfl_sync(0xffffffffu, bb.z, lo);
                bs.w = __shfl_sync(0xffffffffu, bb.w, lo);
                if (qv < total) {
                    int p, c, rr;
                    rec_position(bs, hs, nns, qv - exs, p, c, rr);
                    const long long pos = (long long)offs + p;
                    if (rr < 0) rr = __ldg(&a.idx[pos]) & (NT - 1);
                    const double av = val ? (double)__ldg(&val[pos]) : 1.0;
                    const double xv = __ldcg(&a.L.t_xv[(long long)ss * NT + c]);
                    const long long rc = trs >= 0 ? (long long)trs * NT + rr : ~((long long)(~trs) * NT + rr);
                    frp = contribute<SR, PB>(a, s_hacc, s_hbits, ps, rc, av, xv);
                }
                touch(a, s_pcnt, frq);  // previous round's result: its atomic had a round to return
                frq = frp;
                frp = -1;
            }
            touch(a, s_pcnt, frq);
        }
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        n_hit += __shfl_xor_sync(0xffffffffu, n_hit, o);
        n_hcol += __shfl_xor_sync(0xffffffffu, n_hcol, o);
        n_mac += __shfl_xor_sync(0xffffffffu, n_mac, o);
        n_ind += __shfl_xor_sync(0xffffffffu, n_ind, o);
    }
    if (tr && tid == 0) tr[4] = globaltimer_ns();
    if (lane == 0) {
        s_acct[wid][0] = n_hit;
        s_acct[wid][1] = n_hcol;
        s_acct[wid][2] = n_mac;
        s_acct[wid][3] = n_ind;
    }
    __syncthreads();
    if constexpr (PB) {
        pb_flush<SR>(a, ps, s_hacc, s_hbits, n_slots, s_bhist, s_bbase, s_brank, s_perm, err, s_acct, s_scan, tr);
        if (tr && tid == 0) tr[7] = globaltimer_ns();
        grid_sync_f(&a.cnt->bar, target, tr ? tr + 5 : nullptr);
        if (stamp) ts[3] = globaltimer_ns();
        if (stamp) ts[4] = globaltimer_ns();
        pb_emit<SR, XV>(a, err, s_scan, s_dyn, n_slots, tr);
        if (b == 0 && tid == 0) {
            a.hm->err = err ? 1 : 0;
            // every CTA read err / resv_* after barrier 1
            a.cnt->err = 0;
            a.cnt->resv_t = 0;
            a.cnt->resv_s = 0;
        }
        if (b == G - 1 && tid == 0 && a.tring) ts[5] = globaltimer_ns();
        if (tr && tid == 0) tr[9] = globaltimer_ns();
        return;
    } else {
    // privatised hot rows: one global atomic per (CTA, touched hot row)
#ifdef TSMV_EXP_NO_FLUSH
    if (false) {
#else
    if (!err) {
#endif
        // CTAs start at different slots so that the 148 flushes of one hot row are
        // spread over time instead of queueing on one L2 address together
        // the flush atomics are issued first and their old values consumed after
        // the piece-count flush below, so their round trip overlaps it
        const int rot = (int)(((long long)b * n_slots) / G);
        constexpr int FQ = (HOT_SLOTS + FT - 1) / FT;
        long long row_of[FQ];
        unsigned long long old[FQ];
#pragma unroll
        for (int i = 0; i < FQ; ++i) {
            const int q = tid + i * FT;
            const int sl = q + rot < n_slots ? q + rot : q + rot - n_slots;
            row_of[i] = -1;
            old[i] = 0;
            if (q < n_slots && ((s_hbits[sl >> 5] >> (sl & 31)) & 1u)) {
                const long long row = (long long)s_hlist[sl / NT] * NT + sl % NT;
                row_of[i] = row;
                if constexpr (SR == TSMV_PLUS_TIMES)
                    old[i] = (unsigned long long)__double_as_longlong(atomicAdd(&a.acc[row], s_hacc[sl]));
                else if constexpr (SR == TSMV_MIN_SECOND)
                    old[i] = (unsigned long long)atomicMax((long long *)&a.acc[row],
                                                           (long long)__double_as_longlong(s_hacc[sl]));
                else
                    old[i] = atomicExch((unsigned long long *)&a.acc[row], 0ull);
            }
        }
        if (tid < 4) {
            long long sum = 0;
            for (int w = 0; w < NWF; ++w) sum += s_acct[w][tid];
            a.acct[b * 4 + tid] = sum;
        }
        // piece counts of the rows this CTA touched first in B (s_pcnt is complete:
        // every touch of B happened before the __syncthreads above)
        for (int q = tid; q < a.n_pieces; q += FT)
            if (s_pcnt[q]) atomicAdd(&a.pc[q], s_pcnt[q]);
#pragma unroll
        for (int i = 0; i < FQ; ++i) {
            if (row_of[i] >= 0 && old[i] == EMPTY) {
                const long long row = row_of[i];
                atomicOr(&a.rowbits[row >> 5], 1u << (row & 31));
                atomicAdd(&a.pc[(row >> 5) >> a.ps_log], 1u);
            }
        }
    } else if (tid < 4) {
        long long sum = 0;
        for (int w = 0; w < NWF; ++w) sum += s_acct[w][tid];
        a.acct[b * 4 + tid] = sum;
    }
    if (tr && tid == 0) tr[7] = globaltimer_ns();
    grid_sync_f(&a.cnt->bar, target, tr ? tr + 5 : nullptr);
    if (stamp) ts[3] = globaltimer_ns();

    // ------------------------------------------------------------ phase C (a6)
    // y compaction from the touched bitmap and the piece counts (emit_pieces,
    // spmspv_common.cuh); phase-B windows are free now and hold its dense-word lists
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
        ea.hy_idx = a.hy_idx;
        ea.hy_val = a.hy_val;
        if (stamp) ts[4] = globaltimer_ns();
        emit_pieces<SR, XV, FT, KP, MAXG, SPW, BATCH>(ea, s_scan, s_pbase, s_ex0, s_tot, s_nd, s_win, s_winb,
                                                       reinterpret_cast<unsigned *>(s_winx));
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
    }
    if (tr && tid == 0) tr[9] = globaltimer_ns();
}

template <class AV, class XV, bool PB> void *pick_sr_flat(int sr) {
    if (sr == TSMV_PLUS_TIMES) return (void *)k_spmspv_flat<AV, XV, TSMV_PLUS_TIMES, PB>;
    if (sr == TSMV_OR_AND) return (void *)k_spmspv_flat<AV, XV, TSMV_OR_AND, PB>;
    return (void *)k_spmspv_flat<AV, XV, TSMV_MIN_SECOND, PB>;
}
void *pick_flat(bool f32, int sr, bool pb = false) {
    if (pb) return f32 ? pick_sr_flat<float, float, true>(sr) : pick_sr_flat<double, double, true>(sr);
    return f32 ? pick_sr_flat<float, float, false>(sr) : pick_sr_flat<double, double, false>(sr);
}

constexpr size_t FLAT_DYN = FLAT_DYN_B0 + MAXG * KP * 4;
// dynamic shared memory of the bucketed variant: the whole opt-in maximum less the
// kernel's static shared memory (set once)
size_t g_pb_dyn = 0;

void flat_set_smem() {
    static bool done = false;
    if (done) return;
    int dev = 0, optin = 0;
    TSMV_CUDA(cudaGetDevice(&dev));
    TSMV_CUDA(cudaDeviceGetAttribute(&optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev));
    size_t stat = 0;
    for (int f32 = 0; f32 < 2; ++f32)
        for (int sr = 0; sr < 3; ++sr) {
            TSMV_CUDA(cudaFuncSetAttribute(pick_flat(f32, sr), cudaFuncAttributeMaxDynamicSharedMemorySize,
                                           (int)FLAT_DYN));
            cudaFuncAttributes fa;
            TSMV_CUDA(cudaFuncGetAttributes(&fa, pick_flat(f32, sr, true)));
            stat = std::max(stat, (size_t)fa.sharedSizeBytes);
        }
    g_pb_dyn = ((size_t)optin > stat + 1024 ? (size_t)optin - stat - 1024 : 0) & ~(size_t)15;
    for (int f32 = 0; f32 < 2; ++f32)
        for (int sr = 0; sr < 3; ++sr)
            TSMV_CUDA(cudaFuncSetAttribute(pick_flat(f32, sr, true), cudaFuncAttributeMaxDynamicSharedMemorySize,
                                           (int)g_pb_dyn));
    done = true;
}

template <class V>
__global__ void k_build_rec64(const TileDesc *__restrict__ desc, const uint8_t *__restrict__ cstart,
                              const uint8_t *__restrict__ idx, const V *__restrict__ val, int64_t T,
                              TileRec64 *__restrict__ rec) {
    constexpr int INL = 32 / (int)sizeof(V);
    for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < T; t += (int64_t)gridDim.x * blockDim.x) {
        const TileDesc d = desc[t];
        TileRec64 r;
        r.off = (uint32_t)d.off;
        r.trow = d.trow;
        r.nnz = (uint32_t)d.nnz;
        r.pad = 0;
        uint32_t w[4];
        for (int q = 0; q < 4; ++q) {
            uint32_t x = 0;
            for (int i = 0; i < 4; ++i) {
                const int k = 4 * q + i;
                const uint32_t by = d.nnz <= 16 ? (k < d.nnz ? idx[d.off + k] : 0xffu) : cstart[t * 16 + k];
                x |= by << (8 * i);
            }
            w[q] = x;
        }
        r.b = make_uint4(w[0], w[1], w[2], w[3]);
        V vv[INL];
        for (int i = 0; i < INL; ++i) vv[i] = (val && i < d.nnz && d.nnz <= INL) ? val[d.off + i] : (V)0;
        memcpy(&r.v[0], vv, 32);
        rec[t] = r;
    }
}

__global__ void k_build_colinfo(const long long *__restrict__ sptr, const long long *__restrict__ tptr, int64_t n,
                                int64_t nTC, ColInfo *__restrict__ ci) {
    for (int64_t j = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; j <= n; j += (int64_t)gridDim.x * blockDim.x) {
        ColInfo c;
        c.sbeg = sptr[j];
        const int64_t J = j >> 4;
        c.tinfo = J < nTC ? (((unsigned long long)tptr[J] << 24) | (unsigned long long)(tptr[J + 1] - tptr[J])) : 0ull;
        ci[j] = c;
    }
}

}  // namespace

bool flat_supported(const tsmv_ctx *c) { return c->use_flat; }

namespace {
__global__ void k_fill_u64(unsigned long long *p, long long n, unsigned long long v) {
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x)
        p[i] = v;
}
}  // namespace

// Decide (once, at create) whether the context uses the flat kernel, and set the
// accumulator to its EMPTY encoding (the round-1 fused kernel uses 0).
void flat_init(tsmv_ctx *c, cudaStream_t st) {
    c->use_flat = c->nt == 16 && c->P.rec.p != nullptr && !getenv("TSMV_FUSED_V6");
    if (!c->use_flat || c->m == 0) return;
    const int blocks = (int)std::min<int64_t>((c->m + 255) / 256, 148 * 8);
    k_fill_u64<<<blocks, 256, 0, st>>>(c->acc.as<unsigned long long>(), c->m, EMPTY);
    TSMV_CUDA(cudaGetLastError());
}

void build_rec64(tsmv_ctx *c, TileSet &S, cudaStream_t st) {
    // limits of the packed fields: u32 nonzero offsets, 24-bit tile counts per tile
    // column, 40-bit tile ids
    if (c->nt != 16 || S.T == 0 || S.dense_nnz >= (1ll << 32) || S.nTR >= (1ll << 24) || S.T >= (1ll << 40))
        return;
    S.rec.alloc((size_t)S.T * sizeof(TileRec64));
    const int blocks = (int)std::min<int64_t>((S.T + 255) / 256, 148 * 16);
    if (c->dtype == TSMV_F32)
        k_build_rec64<float><<<blocks, 256, 0, st>>>(S.desc.as<TileDesc>(), S.cstart.as<uint8_t>(),
                                                      S.idx.as<uint8_t>(), S.has_vals ? S.val.as<float>() : nullptr,
                                                      S.T, S.rec.as<TileRec64>());
    else
        k_build_rec64<double><<<blocks, 256, 0, st>>>(S.desc.as<TileDesc>(), S.cstart.as<uint8_t>(),
                                                       S.idx.as<uint8_t>(), S.has_vals ? S.val.as<double>() : nullptr,
                                                       S.T, S.rec.as<TileRec64>());
    TSMV_CUDA(cudaGetLastError());
    S.colinfo.alloc((size_t)(S.dimC + 1) * sizeof(ColInfo));
    const int cb = (int)std::min<int64_t>((S.dimC + 256) / 256, 148 * 16);
    k_build_colinfo<<<cb, 256, 0, st>>>(S.sptr.as<long long>(), S.ptr.as<long long>(), S.dimC, S.nTC,
                                        S.colinfo.as<ColInfo>());
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
        F.t_xv.alloc(segs * 16 * 8);
        F.s_beg.alloc((cap + 1) * 8);
        F.s_wpre.alloc((cap + 1) * 8);
        F.s_x.alloc((cap + 1) * 8);
        F.cap_ent = cap;
    }
    if (!F.Ct.p) {
        F.Ct.alloc(((c->P.T >> TL) + 2) * 4);
        F.Cs.alloc(((c->P.side_nnz >> SL) + 2) * 4);
        F.hits.alloc((size_t)(c->P.T + (1ll << TL) * (c->flat_blocks + 2)) * 16);
        F.pcnt.alloc((size_t)2 * MAXG * KP * 4);  // u32[2][MAXG * KP]: piece counts, double-buffered
        TSMV_CUDA(cudaMemset(F.pcnt.p, 0, F.pcnt.bytes));
    }
}

FlatListsView flat_view(tsmv_ctx *c) {
    FlatListsView v;
    v.t_beg = c->FL.t_beg.as<long long>();
    v.t_wpre = c->FL.t_wpre.as<long long>();
    v.t_xm = c->FL.t_xm.as<unsigned>();
    v.t_J = c->FL.t_J.as<int>();
    v.t_xv = c->FL.t_xv.as<double>();
    v.s_beg = c->FL.s_beg.as<long long>();
    v.s_wpre = c->FL.s_wpre.as<long long>();
    v.s_x = c->FL.s_x.as<double>();
    v.Ct = c->FL.Ct.as<int>();
    v.Cs = c->FL.Cs.as<int>();
    v.hits = c->FL.hits.as<uint4>();
    v.pcnt = c->FL.pcnt.as<long long>();
    v.xd = c->xdense.as<double>();
    return v;
}

namespace {
// nonzeros of the rows of every bucket (block per bucket)
__global__ void k_pb_bucket_nnz(const int32_t *__restrict__ indeg, long long m, int bl, long long *__restrict__ out) {
    __shared__ long long s[8];
    const long long r0 = (long long)blockIdx.x << bl, r1 = min(m, r0 + (1ll << bl));
    long long v = 0;
    for (long long r = r0 + threadIdx.x; r < r1; r += blockDim.x) v += indeg[r];
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    if ((threadIdx.x & 31) == 0) s[threadIdx.x >> 5] = v;
    __syncthreads();
    if (threadIdx.x == 0) {
        long long t = 0;
        for (int w = 0; w < (int)(blockDim.x >> 5); ++w) t += s[w];
        out[blockIdx.x] = t;
    }
}
}  // namespace

// Bucketed variant: buckets of 2^bl rows (bl in [10, 14], the smallest giving
// <= 512 buckets), staging regions sized by the nonzeros of each bucket's rows
// (a call stages at most one product per nonzero), allocated on first use.
static bool pb_setup(tsmv_ctx *c, cudaStream_t st) {
    if (c->pb_state) return c->pb_state > 0;
    c->pb_state = -1;
    if (c->m == 0 || c->flat_blocks == 0) return false;
    flat_set_smem();
    int bl = 10;
    while (bl < 14 && ((c->m + (1ll << bl) - 1) >> bl) > 512) ++bl;
    if (const char *e = getenv("TSMV_PB_BL")) bl = std::min(14, std::max(10, atoi(e)));
    const long long NB = (c->m + (1ll << bl) - 1) >> bl;
    if (NB > 4ll * FT) return false;
    const size_t b0 = pb_align(FLAT_DYN_B0) + (size_t)NB * 12;
    const size_t cneed = ((size_t)8 << bl) + ((size_t)8 << bl) / 32 + (size_t)NB * 8;
    if (g_pb_dyn < b0 + 16 * 1024 || g_pb_dyn < cneed) return false;
    c->pb_bl = bl;
    c->pb_nb = (int)NB;
    c->pb_cap = (int)std::min<size_t>(65535, (g_pb_dyn - b0) / 16);
    if (const char *e = getenv("TSMV_PB_CAP")) c->pb_cap = std::max(1, std::min(c->pb_cap, atoi(e)));  // tests: overflow
    DevBuf sums;
    sums.alloc(NB * 8);
    k_pb_bucket_nnz<<<(unsigned)NB, 256, 0, st>>>(c->indeg.as<int32_t>(), c->m, bl, sums.as<long long>());
    TSMV_CUDA(cudaGetLastError());
    std::vector<long long> h(NB + 1, 0);
    TSMV_CUDA(cudaMemcpyAsync(h.data() + 1, sums.p, NB * 8, cudaMemcpyDeviceToHost, st));
    TSMV_CUDA(cudaStreamSynchronize(st));
    for (long long q = 0; q < NB; ++q) h[q + 1] += h[q];
    c->pb_rs.alloc((NB + 1) * 8);
    TSMV_CUDA(cudaMemcpyAsync(c->pb_rs.p, h.data(), (NB + 1) * 8, cudaMemcpyHostToDevice, st));
    const long long cap = std::max<long long>(h[NB], 1);
    c->pb_row.alloc(cap * 4);
    c->pb_val.alloc(cap * 8);
    c->pb_cnt.alloc(2 * NB * 4);
    c->pb_agg.alloc((size_t)2 * MAXG * 8);
    // hot rows: per-CTA partial slots, and the slots of every bucket
    const int n_slots = c->P.hot_list ? c->n_hot * 16 : 0;
    c->pb_hp.alloc((size_t)std::max(1, MAXG * n_slots) * 8);
    c->pb_hr.alloc((size_t)std::max(1, n_slots) * 12);
    TSMV_CUDA(cudaMemset(c->pb_hr.p, 0, c->pb_hr.bytes));
    std::vector<int> hs, hso(NB + 1, 0);
    if (n_slots) {
        std::vector<int32_t> hl(c->n_hot);
        TSMV_CUDA(cudaMemcpy(hl.data(), c->P.hot_list, c->n_hot * 4, cudaMemcpyDeviceToHost));
        std::vector<std::pair<long long, int>> rows;
        for (int sl = 0; sl < n_slots; ++sl) {
            const long long row = (long long)hl[sl / 16] * 16 + sl % 16;
            if (row < c->m) rows.push_back({row, sl});
        }
        std::sort(rows.begin(), rows.end());
        for (auto &r : rows) {
            hs.push_back(r.second);
            hso[(r.first >> bl) + 1]++;
        }
        for (long long q = 0; q < NB; ++q) hso[q + 1] += hso[q];
    }
    c->pb_hs.alloc(std::max<size_t>(hs.size(), 1) * 4);
    c->pb_hso.alloc((NB + 1) * 4);
    if (!hs.empty()) TSMV_CUDA(cudaMemcpy(c->pb_hs.p, hs.data(), hs.size() * 4, cudaMemcpyHostToDevice));
    TSMV_CUDA(cudaMemcpy(c->pb_hso.p, hso.data(), (NB + 1) * 4, cudaMemcpyHostToDevice));
    TSMV_CUDA(cudaMemsetAsync(c->pb_cnt.p, 0, c->pb_cnt.bytes, st));
    TSMV_CUDA(cudaMemsetAsync(c->pb_agg.p, 0, c->pb_agg.bytes, st));
    TSMV_CUDA(cudaStreamSynchronize(st));
    c->pb_state = 1;
    return true;
}

// Bucketed variant only when forced (TSMV_SPMSPV_KERNEL=pb): measured slower
// than the plain kernel at every density tried, kept as an
// experiment with its parity tests.
static bool use_pb(tsmv_ctx *c, long long k, cudaStream_t st) {
    (void)k;
    const char *f = getenv("TSMV_SPMSPV_KERNEL");
    return f && f[0] == 'p' && pb_setup(c, st);
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
    a.rec = c->P.rec.as<TileRec64>();
    a.colinfo = c->P.colinfo.as<ColInfo>();
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
    {
        // pieces of 2^ps_log bitmap words, at most G * KP of them (phase C)
        const long long per = (a.W + (long long)c->flat_blocks * KP - 1) / ((long long)c->flat_blocks * KP);
        int lg = 5;
        while ((1ll << lg) < per) ++lg;
        a.ps_log = lg;
        a.n_pieces = (int)((a.W + (1ll << lg) - 1) >> lg);
        unsigned *pc = c->FL.pcnt.as<unsigned>();
        const int cur = (int)(c->flat_calls & 1);
        a.pc = pc + (size_t)cur * MAXG * KP;
        a.pc_next = pc + (size_t)(1 - cur) * MAXG * KP;
    }
    const bool pb = use_pb(c, k, st);
    if (pb) {
        const long long NB = c->pb_nb;
        const int cur = (int)(c->pb_calls & 1);
        a.pb_rs = c->pb_rs.as<long long>();
        a.pb_row = c->pb_row.as<unsigned>();
        a.pb_val = c->pb_val.as<unsigned long long>();
        a.pb_cnt = c->pb_cnt.as<unsigned>() + cur * NB;
        a.pb_cnt_next = c->pb_cnt.as<unsigned>() + (1 - cur) * NB;
        a.pb_agg = c->pb_agg.as<unsigned long long>();
        a.pb_pu = a.pb_agg + MAXG;
        a.pb_hp = c->pb_hp.as<unsigned long long>();
        a.pb_hr = c->pb_hr.as<unsigned long long>();
        a.pb_hre = reinterpret_cast<unsigned *>(a.pb_hr + std::max(1, (c->P.hot_list ? c->n_hot : 0) * 16));
        a.pb_hs = c->pb_hs.as<int>();
        a.pb_hso = c->pb_hso.as<int>();
        a.pb_epoch = (unsigned)(c->pb_calls % 0x7fffffffll) + 1u;
        a.pb_bl = c->pb_bl;
        a.pb_nb = c->pb_nb;
        a.pb_cap = c->pb_cap;
        a.pb_ovh = 1ll << (c->pb_bl - 1);
        if (const char *e = getenv("TSMV_PB_OVH")) a.pb_ovh = atoll(e);
        c->pb_calls++;
    } else {
        a.pb_rs = nullptr;
        a.pb_row = nullptr;
        a.pb_val = nullptr;
        a.pb_cnt = a.pb_cnt_next = nullptr;
        a.pb_agg = a.pb_pu = a.pb_hp = a.pb_hr = nullptr;
        a.pb_hre = nullptr;
        a.pb_hs = a.pb_hso = nullptr;
        a.pb_epoch = 0;
        a.pb_bl = a.pb_nb = a.pb_cap = 0;
        a.pb_ovh = 0;
        c->flat_calls++;
    }
    a.cnt = c->counters.as<Counters>();
    a.hm = c->hcnt_dev;
    a.bar_base = c->bar_base;
    a.tring = c->timing ? c->tring.as<unsigned long long>() : nullptr;
    a.tslot = c->tcalls;
    a.hot_list = c->P.hot_list;
    a.n_hot = c->P.hot_list ? c->n_hot : 0;
    a.trace = (unsigned long long *)c->trace;
    a.hy_idx = nullptr;
    a.hy_val = nullptr;
    if (!pb && (c->hy_idx || c->hy_val)) {
        a.hy_idx = c->hy_idx;
        a.hy_val = c->hy_val;
        c->hy_by_kernel = true;
    }
    void *args[] = {&a};
    const int G = c->flat_blocks;
    flat_set_smem();
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(G);
    cfg.blockDim = dim3(FT);
    cfg.dynamicSmemBytes = pb ? g_pb_dyn : FLAT_DYN;
    cfg.stream = st;
    cudaLaunchAttribute at[2];
    at[0].id = cudaLaunchAttributeCooperative;
    at[0].val.cooperative = 1;
    cfg.numAttrs = 1;
    if (c->persist_bytes && !pb) {
        at[1].id = cudaLaunchAttributeAccessPolicyWindow;
        at[1].val.accessPolicyWindow.base_ptr = c->acc.p;
        at[1].val.accessPolicyWindow.num_bytes = c->persist_bytes;
        at[1].val.accessPolicyWindow.hitRatio = c->persist_ratio;
        at[1].val.accessPolicyWindow.hitProp = cudaAccessPropertyPersisting;
        at[1].val.accessPolicyWindow.missProp = cudaAccessPropertyStreaming;
        cfg.numAttrs = 2;
    }
    cfg.attrs = at;
    TSMV_CUDA(cudaLaunchKernelExC(&cfg, pick_flat(f32, sr, pb), args));
    c->bar_base += 2ull * (unsigned long long)G;
    c->last_blocks = G;
    if (c->timing) c->tcalls++;
}

}  // namespace tsmv
