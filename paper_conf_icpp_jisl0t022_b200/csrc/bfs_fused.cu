// bfs_fused.cu -- single-GPU TileBFS as ONE cooperative persistent kernel
// (Alg 3, Sec 3.4).
//
// The level loop runs on the device: per level
//   S  frontier scan: each CTA takes a slice of the nt-segments of F, counts
//      (segments with tiles, tile work, vertices with side work, side work,
//      |F|, m_f = sum outdeg(F), sum indeg(F)) and clears the bitmap of the
//      previous frontier (it becomes the next-frontier target);
//   -- barrier --  every CTA reduces the per-CTA totals itself, takes the same
//      direction decision (reading R9: m_f vs m_u / alpha, |F|/n vs 0.01) and
//      writes its part of the work lists;
//   -- barrier --
//   E  expand with the chosen kernel: Push-CSC (Alg 5, load-balanced chunks
//      over the frontier's tile columns + side columns), Push-CSR (Alg 6,
//      tile-parallel + side push) or Pull-CSC (Alg 7, warp per row tile with
//      early exit + side pull);
//   -- barrier --
// until the frontier is empty.  No host round trip per level (the per-level
// kernels of bfs.cu remain for the distributed driver).
//
// List-driven push levels (high-diameter graphs: stencils, bands, late R-MAT
// levels).  While the rule picks Push-CSC and no frontier vertex has more than
// LIST_MAXW items of push work, a level is ONE phase and ONE grid barrier: a
// group of G lanes per frontier vertex u (taken from the vertex list of the
// level) ORs plane c = u % nt of every tile of u's tile column into V and walks
// u's side column; each newly discovered vertex gets its level, is appended to
// the next level's list through a per-CTA shared-memory queue and adds its
// out-degree / in-degree / push work to the next level's counters (three
// rotating slots).  The first level that needs the bitmap form (Pull-CSC,
// Push-CSR or a heavy vertex) writes the list into the frontier bitmap and
// continues with the 3-barrier scan levels above.
#include "bfs_dev.cuh"

namespace tsmv {

namespace {

constexpr int BFB = 512;  // threads per CTA
constexpr int MAXBG = 320;  // max CTAs of the persistent grid (2 per SM up to 160 SMs; partial sums read at once)
constexpr int LIST_MAXW = 512;   // list levels only while every frontier vertex has <= this much push work
#ifndef TSMV_QCAP
#define TSMV_QCAP 2048
#endif
constexpr int QCAP = TSMV_QCAP;  // per-CTA shared-memory queue of discovered vertices
constexpr int SOLO_QS = BFB;     // solo levels: frontier records in shared memory (one per thread)
constexpr int SOLO_ITEMS = 4 * BFB;  // solo while the level's push work <= 4 items per thread

struct BfsFusedArgs {
    BfsTiles P, Q;
    BfsView B;            // V, F (=F0), Fn (=F1), levels, n, m
    const int *outdeg, *indeg;
    ListsView Lv;
    long long *partials;  // [G][8]
    Counters *cnt;
    Counters *hm;         // mapped: fsize (levels), reached, edges
    int *dir_out;         // [TSMV_MAX_LEVELS] direction of level L (stats; written for L < TSMV_MAX_LEVELS)
    long long *front_out; // [TSMV_MAX_LEVELS] |F| of level L
    unsigned long long *tlv_out;  // [TSMV_MAX_LEVELS + 1] %globaltimer when level L's expansion is decided
    long long source, nnz, nseg, NW, nTR_local, max_levels;
    double alpha, dens;
    double alpha_burst, growth;   // reading R9' (explosive levels)
    long long fprev0;             // |F| of the level before level0 (resume), 0 = none
    int force;
    unsigned long long bar_base;
    // resume / hand-off: the kernel stops before expanding a
    // Pull-CSC level when stop_on_pull is set; the host runs that level with the
    // high-occupancy per-level kernels and resumes the kernel afterwards
    int resume, stop_on_pull;
    long long level0, mu0, reached0, edges0;
    // list-driven push levels
    const int *lwork;
    int *bq0, *bq1;
    long long *lslots;   // [3][4] slots, [12..15] profiling, [16] solo release flag, [17..20] solo state
    int use_list, use_solo;
    int no_relist;       // TSMV_BFS_NO_RELIST: scan levels never convert back to list levels (A/B)
    int stop_on_bulk;    // heavy bulk Push-CSC levels go to the host kernels (TSMV_BFS_BULK_HOST=0: stay)
    long long bulk_stop_min;
    int qcap;                 // usable entries of the shared-memory queue (<= QCAP; TSMV_BFS_QCAP tests the overflow path)
    int wide_in_kernel;       // pull levels with m_u < nnz / 4 stay in the kernel (wide pull)
    long long wide_cap;       // ... unless m_u > wide_cap (r2: large graphs)
    int bulk_push;            // heavy Push-CSC levels in bulk mode (r2)
    // r2: L2 warm-up of the push structures + degrees (graphs whose structures fit
    // in half the L2): bulk L2 prefetches by every CTA before the first level, so the
    // latency-bound list / solo levels of high-diameter graphs hit L2, not HBM
    const void *pf_p[8];
    long long pf_b[8];
    int pf_n;
};
constexpr long long PF_CHUNK = 8192;

struct SoloShared {
    int cnt, W;
    unsigned long long mf, din;
    int maxw, pad2;
};

struct ListShared {
    int qn, base, maxw, pad;
    unsigned long long mf, din;
    int q[QCAP];
};

// Discovery in a list level: V bits, levels and the CTA's queue.  Degrees are
// read later, in parallel over the queue (list_flush), not in this serial loop.
template <int NT>
__device__ __forceinline__ void discover_list(const BfsFusedArgs &a, const BfsView &B, long long gseg,
                                              typename Tr<NT>::word_t bits, ListShared &sh, int *Qn,
                                              long long *slot_n) {
    using word_t = typename Tr<NT>::word_t;
    const word_t old = seg_or<NT>(B.V, gseg, bits);
    word_t nw = bits & ~old;
    if (!nw) return;
    int p = atomicAdd(&sh.qn, popc_w(nw));
    while (nw) {
        const int r = ffs_w(nw);
        nw &= nw - 1;
        const long long v = gseg * NT + r;
        B.levels[v] = B.level + 1;
        if (p < a.qcap) {
            sh.q[p] = (int)v;
        } else {  // queue full: straight to the global list and counters
            const unsigned long long gp = atomicAdd((unsigned long long *)&slot_n[0], 1ull);
            Qn[gp] = (int)v;
            atomicAdd((unsigned long long *)&slot_n[1], (unsigned long long)a.outdeg[v]);
            atomicAdd((unsigned long long *)&slot_n[2], (unsigned long long)a.indeg[v]);
            atomicMax(&slot_n[3], (long long)a.lwork[v]);
        }
        ++p;
    }
}

// End of a list level in one CTA: reserve the CTA's range of the next list,
// copy the queue there and add its degrees / max work to the next slot.
__device__ __forceinline__ void list_flush(const BfsFusedArgs &a, ListShared &sh, int *Qn, long long *slot_n,
                                           int tid, int lane) {
    __syncthreads();
    const int qn = min(sh.qn, a.qcap);
    if (qn == 0) return;  // uniform: no __syncthreads skipped by part of the CTA
    if (tid == 0) sh.base = (int)atomicAdd((unsigned long long *)&slot_n[0], (unsigned long long)qn);
    __syncthreads();
    unsigned long long mf = 0, din = 0;
    int mx = 0;
    for (int i = tid; i < qn; i += BFB) {
        const int v = sh.q[i];
        Qn[sh.base + i] = v;
        mf += (unsigned long long)a.outdeg[v];
        din += (unsigned long long)a.indeg[v];
        mx = max(mx, a.lwork[v]);
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        mf += __shfl_xor_sync(0xffffffffu, mf, o);
        din += __shfl_xor_sync(0xffffffffu, din, o);
        mx = max(mx, __shfl_xor_sync(0xffffffffu, mx, o));
    }
    if (lane == 0 && mf + din + (unsigned long long)mx) {
        atomicAdd(&sh.mf, mf);
        atomicAdd(&sh.din, din);
        atomicMax(&sh.maxw, mx);
    }
    __syncthreads();
    if (tid == 0) {
        atomicAdd((unsigned long long *)&slot_n[1], sh.mf);
        atomicAdd((unsigned long long *)&slot_n[2], sh.din);
        atomicMax(&slot_n[3], (long long)sh.maxw);
    }
}

// One list level: group of G lanes per frontier vertex.  A group takes LR
// vertices at a time and issues each dependent step (list entry -> column
// ranges -> first plane word / side row -> V) for all of them before the next,
// so LR chains of loads are in flight per lane instead of one.
#ifndef TSMV_LR
#define TSMV_LR 1
#endif
constexpr int LR = TSMV_LR;

template <int NT>
__device__ __forceinline__ void list_level(const BfsFusedArgs &a, const BfsView &B, const int *Qc, long long fsize,
                                           int G, long long gtid, long long gthreads, ListShared &sh, int *Qn,
                                           long long *slot_n) {
    using word_t = typename Tr<NT>::word_t;
    const word_t *planes = (const word_t *)a.P.planes;
    const long long ngroups = gthreads / G;
    const long long gid = gtid / G;
    const int gl = (int)(gtid % G);
    for (long long i0 = gid; i0 < fsize; i0 += LR * ngroups) {
        long long u[LR], t0[LR], ntl[LR], s0[LR], ns[LR];
#pragma unroll
        for (int r = 0; r < LR; ++r) {
            const long long i = i0 + r * ngroups;
            u[r] = i < fsize ? (long long)__ldcg(&Qc[i]) : -1;
        }
#pragma unroll
        for (int r = 0; r < LR; ++r) {
            t0[r] = ntl[r] = s0[r] = ns[r] = 0;
            if (u[r] >= 0) {
                const long long J = u[r] / NT;
                t0[r] = __ldg(&a.P.ptr[J]);
                ntl[r] = __ldg(&a.P.ptr[J + 1]) - t0[r];
                s0[r] = __ldg(&a.P.sptr[u[r]]);
                ns[r] = __ldg(&a.P.sptr[u[r] + 1]) - s0[r];
            }
        }
        // first item of every vertex: loads for all LR vertices, then the ORs
        word_t w[LR];
        long long seg[LR];
#pragma unroll
        for (int r = 0; r < LR; ++r) {
            w[r] = 0;
            seg[r] = 0;
            if (u[r] >= 0) {
                if (gl < ntl[r]) {
                    const long long t = t0[r] + gl;
                    w[r] = __ldg(&planes[(long long)(u[r] % NT) * a.P.T + t]);
                    seg[r] = __ldg(&a.P.trow[t]);
                } else if (gl < ntl[r] + ns[r]) {
                    const long long v = decode_row<NT>(__ldg(&a.P.srow[s0[r] + (gl - ntl[r])]), a.P.hot_list);
                    w[r] = (word_t)1 << (v % NT);
                    seg[r] = v / NT;
                }
            }
        }
#pragma unroll
        for (int r = 0; r < LR; ++r)
            if (w[r]) discover_list<NT>(a, B, seg[r], w[r], sh, Qn, slot_n);
        // remaining items (vertices with more than G items of work)
#pragma unroll 1
        for (int r = 0; r < LR; ++r) {
            const int c = (int)(u[r] % NT);
            for (long long k = gl + G; k < ntl[r] + ns[r]; k += G) {
                if (k < ntl[r]) {
                    const long long t = t0[r] + k;
                    const word_t ww = planes[(long long)c * a.P.T + t];
                    if (ww) discover_list<NT>(a, B, (long long)a.P.trow[t], ww, sh, Qn, slot_n);
                } else {
                    const long long v = decode_row<NT>(a.P.srow[s0[r] + (k - ntl[r])], a.P.hot_list);
                    discover_list<NT>(a, B, v / NT, (word_t)1 << (v % NT), sh, Qn, slot_n);
                }
            }
        }
    }
}

// Chunk -> list-entry map for an entry owning work items [w0, w0 + w): short runs
// by the calling thread, runs over 8 chunks (hub columns: thousands) queued for a
// warp of the CTA (one thread used to write a hub's whole map serially).
constexpr int HVQ = 64;
__device__ __forceinline__ void put_chunks_q(int *C, long long w0, long long w, int entry, int kind,
                                             long long (*hv)[3], int *nhv) {
    const long long c0 = (w0 + CHUNK - 1) >> CHUNK_LOG, c1 = (w0 + w + CHUNK - 1) >> CHUNK_LOG;
    if (c1 - c0 > 8) {
        const int q = atomicAdd(nhv, 1);
        if (q < HVQ) {
            hv[q][0] = c0;
            hv[q][1] = c1;
            hv[q][2] = ((long long)kind << 32) | (unsigned)entry;
            return;
        }
    }
    for (long long ch = c0; ch < c1; ++ch) C[ch] = entry;
}

template <int NT>
__device__ __forceinline__ void seg_counts(const BfsFusedArgs &a, const uint32_t *F, long long J, long long *v) {
    using word_t = typename Tr<NT>::word_t;
    const word_t bits = seg_bits<NT>(F, J);
    if (!bits) return;
    if constexpr (NT == 16) {
        // 16 out-degrees, in-degrees and 17 side starts of the segment are
        // contiguous (arrays padded to whole segments): vector loads, one latency
        const long long wt = a.P.ptr[J + 1] - a.P.ptr[J];
        v[0] += wt > 0;
        v[1] += wt;
        v[4] += popc_w(bits);
        const long long v0 = J * 16;
        int od[16], id[16];
        long long sp[17];
#pragma unroll
        for (int i = 0; i < 4; ++i) {
            const int4 t = __ldg(reinterpret_cast<const int4 *>(a.outdeg + v0) + i);
            od[4 * i] = t.x, od[4 * i + 1] = t.y, od[4 * i + 2] = t.z, od[4 * i + 3] = t.w;
        }
        if (v0 + 16 <= a.B.m_local) {
#pragma unroll
            for (int i = 0; i < 4; ++i) {
                const int4 t = __ldg(reinterpret_cast<const int4 *>(a.indeg + v0) + i);
                id[4 * i] = t.x, id[4 * i + 1] = t.y, id[4 * i + 2] = t.z, id[4 * i + 3] = t.w;
            }
        } else {
#pragma unroll
            for (int r = 0; r < 16; ++r) id[r] = v0 + r < a.B.m_local ? __ldg(a.indeg + v0 + r) : 0;
        }
#pragma unroll
        for (int i = 0; i < 8; ++i) {
            const longlong2 t = __ldg(reinterpret_cast<const longlong2 *>(a.P.sptr + v0) + i);
            sp[2 * i] = t.x, sp[2 * i + 1] = t.y;
        }
        sp[16] = __ldg(a.P.sptr + v0 + 16);
#pragma unroll
        for (int r = 0; r < 16; ++r) {
            if ((bits >> r) & 1u) {
                const long long ws = sp[r + 1] - sp[r];
                v[2] += ws > 0;
                v[3] += ws;
                v[5] += od[r];
                v[6] += id[r];
            }
        }
        return;
    }
    const long long wt = a.P.ptr[J + 1] - a.P.ptr[J];
    v[0] += wt > 0;
    v[1] += wt;
    v[4] += popc_w(bits);
    word_t b = bits;
    while (b) {
        const int r = ffs_w(b);
        b &= b - 1;
        const long long u = J * NT + r;
        const long long ws = a.P.sptr[u + 1] - a.P.sptr[u];
        v[2] += ws > 0;
        v[3] += ws;
        v[5] += a.outdeg[u];
        v[6] += a.indeg[u];
    }
}

// Solo levels (session 3; r2 restructured): while the frontier is small, CTA 0
// alone runs the list levels with the level in shared memory and __syncthreads
// instead of grid barriers; the other CTAs wait on a release flag.  r2: a
// frontier entry is a 16-byte record {v, tile start, side start, tile count,
// side count} built when v is discovered, in the same pass (and the same memory
// latency) as v's degrees, and the level's push work is flattened into an item
// map (item -> entry), so a level is
//   items (smem) -> up to 4 plane / side words per thread, loads issued together
//   -> atomicOr V -> next ids (smem) -> __syncthreads
//   -> per new vertex: degrees + column starts (one latency) -> records, block
//      scan of the work, item map -> __syncthreads,
// three dependent global round trips per level instead of seven.  On exit the
// next frontier is left in the global list and its counter slot, exactly as a
// grid list level leaves it.  Entry: level L already counted (mu, reached,
// edges, dir_out); |F| <= SOLO_QS and |F| x max work <= SOLO_ITEMS.
struct SoloRec {
    int v;
    unsigned t0, s0;              // tile / side starts (< 2^32: use_solo checks)
    unsigned short ntl, ns;       // tile / side counts (<= LIST_MAXW)
};
struct SoloBuf {
    SoloRec rec[SOLO_QS];
    int pre[SOLO_QS];             // exclusive prefix of the entries' work
    int nq[SOLO_QS];              // ids found by the level (next frontier)
    unsigned long long part_mf[BFB / 32], part_din[BFB / 32];
    int part_mx[BFB / 32];
    unsigned short item[SOLO_ITEMS];
    cub::BlockScan<int, BFB>::TempStorage scan;
};

// records + item map of the n <= SOLO_QS entries ids[0..n); with `stats` also the
// level's degree sums (ss.mf, ss.din) and the maximum work (ss.maxw); ss.W = items
template <int NT>
__device__ void solo_records(const BfsFusedArgs &a, const int *ids, bool ids_global, long long n, SoloBuf &sb,
                             SoloShared &ss, int tid, long long &out_mf, long long &out_din, long long &out_mx) {
    int w = 0;
    unsigned long long mf = 0, din = 0;
    if (tid < n) {
        const int v = ids_global ? __ldcg(&ids[tid]) : ids[tid];
        const long long J = v / NT;
        const long long t0 = a.P.ptr[J], t1 = a.P.ptr[J + 1];
        const long long s0 = a.P.sptr[v], s1 = a.P.sptr[v + 1];
        mf = (unsigned long long)a.outdeg[v];
        din = (unsigned long long)a.indeg[v];
        SoloRec r;
        r.v = v;
        r.t0 = (unsigned)t0;
        r.s0 = (unsigned)s0;
        r.ntl = (unsigned short)min(t1 - t0, 65535LL);
        r.ns = (unsigned short)min(s1 - s0, 65535LL);
        sb.rec[tid] = r;
        w = (int)min((t1 - t0) + (s1 - s0), (long long)INT_MAX / 4);
    }
    {
        // warp partials (no 64-bit shared atomics: they serialised the level)
        int mx = w;
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) {
            mf += __shfl_xor_sync(0xffffffffu, mf, o);
            din += __shfl_xor_sync(0xffffffffu, din, o);
            mx = max(mx, __shfl_xor_sync(0xffffffffu, mx, o));
        }
        if ((tid & 31) == 0) {
            sb.part_mf[tid >> 5] = mf;
            sb.part_din[tid >> 5] = din;
            sb.part_mx[tid >> 5] = mx;
        }
    }
    int pre, tot;
    cub::BlockScan<int, BFB>(sb.scan).ExclusiveSum(w, pre, tot);
    if (tid < n) sb.pre[tid] = pre;
    if (tot <= SOLO_ITEMS)
        for (int k = 0; k < w; ++k) sb.item[pre + k] = (unsigned short)tid;
    if (tid == 0) ss.W = tot;
    __syncthreads();
    // every thread sums the partials itself (broadcast reads, no further barrier)
    unsigned long long smf = 0, sdin = 0;
    int smx = 0;
#pragma unroll
    for (int i = 0; i < BFB / 32; ++i) {
        smf += sb.part_mf[i];
        sdin += sb.part_din[i];
        smx = max(smx, sb.part_mx[i]);
    }
    out_mf = (long long)smf;
    out_din = (long long)sdin;
    out_mx = smx;
}

template <int NT>
__device__ void solo_levels(const BfsFusedArgs &a, BfsView &B, int &level, long long &mu, long long &reached,
                            long long &edges, long long fsize, long long &fprev, SoloBuf &sb, SoloShared &ss,
                            int tid) {
    using word_t = typename Tr<NT>::word_t;
    const word_t *planes = (const word_t *)a.P.planes;
    long long mf2, din2, mx2;
    solo_records<NT>(a, (level & 1) ? a.bq1 : a.bq0, true, fsize, sb, ss, tid, mf2, din2, mx2);
    long long n = fsize;
#ifdef TSMV_SOLO_PROF
    long long pc[5] = {0, 0, 0, 0, 0}, nlev = 0, c0 = clock64(), c1;
#define SOLO_T(i) (c1 = clock64(), pc[i] += c1 - c0, c0 = c1)
#else
#define SOLO_T(i)
#endif
    while (true) {
        B.level = level;
        int *Qn = (level & 1) ? a.bq0 : a.bq1;  // list of level + 1 (overflow beyond SOLO_QS)
        const int W = ss.W;
        __syncthreads();  // every thread has read W before ss is reset
        if (tid == 0) {
            ss.cnt = 0;
            ss.mf = 0;
            ss.din = 0;
            ss.maxw = 0;
        }
        // ---- expand: item e = tid + k * BFB, k < 4 (W <= SOLO_ITEMS = 4 BFB)
        word_t bits[4];
        long long gseg[4];
#pragma unroll
        for (int k = 0; k < 4; ++k) {
            bits[k] = 0;
            gseg[k] = 0;
            const int e = tid + k * BFB;
            if (e < W) {
                const int i = sb.item[e];
                const SoloRec r = sb.rec[i];
                const int kk = e - sb.pre[i];
                const int c = r.v % NT;
                if (kk < r.ntl) {
                    const long long t = (long long)r.t0 + kk;
                    bits[k] = planes[(long long)c * a.P.T + t];
                    gseg[k] = a.P.trow[t];
                } else {
                    const long long v = decode_row<NT>(a.P.srow[(long long)r.s0 + (kk - r.ntl)], a.P.hot_list);
                    bits[k] = (word_t)1 << (v % NT);
                    gseg[k] = v / NT;
                }
            }
        }
        __syncthreads();  // ss reset visible; records / items no longer read after the loads
        SOLO_T(0);
        // all of a thread's atomics first (independent round trips in flight
        // together), then the discoveries
        word_t olds[4];
#pragma unroll
        for (int k = 0; k < 4; ++k) olds[k] = bits[k] ? seg_or<NT>(B.V, gseg[k], bits[k]) : bits[k];
#pragma unroll
        for (int k = 0; k < 4; ++k) {
            word_t nw = bits[k] & ~olds[k];
            if (!nw) continue;
            int p = atomicAdd(&ss.cnt, popc_w(nw));
            while (nw) {
                const int r = ffs_w(nw);
                nw &= nw - 1;
                const long long v = gseg[k] * NT + r;
                B.levels[v] = level + 1;
                if (p < SOLO_QS) sb.nq[p] = (int)v;
                else Qn[p] = (int)v;
                ++p;
            }
        }
        __syncthreads();
        SOLO_T(1);
        const long long n2 = ss.cnt;
        ++level;
        if (n2 <= SOLO_QS) {
            // records of the next level (its degrees in the same pass)
            solo_records<NT>(a, sb.nq, false, n2, sb, ss, tid, mf2, din2, mx2);
            SOLO_T(2);
        } else {
            unsigned long long mf = 0, din = 0;
            int mx = 0;
            for (long long i = tid; i < n2; i += BFB) {
                const int v = i < SOLO_QS ? sb.nq[i] : __ldcg(&Qn[i]);
                mf += (unsigned long long)a.outdeg[v];
                din += (unsigned long long)a.indeg[v];
                mx = max(mx, a.lwork[v]);
            }
#pragma unroll
            for (int o = 16; o > 0; o >>= 1) {
                mf += __shfl_xor_sync(0xffffffffu, mf, o);
                din += __shfl_xor_sync(0xffffffffu, din, o);
                mx = max(mx, __shfl_xor_sync(0xffffffffu, mx, o));
            }
            if ((tid & 31) == 0 && (mf | din | (unsigned long long)mx)) {
                atomicAdd(&ss.mf, mf);
                atomicAdd(&ss.din, din);
                atomicMax(&ss.maxw, mx);
            }
            __syncthreads();
            mf2 = (long long)ss.mf;
            din2 = (long long)ss.din;
            mx2 = ss.maxw;
        }
        const int dir2 =
            n2 > 0 ? choose_dir_dev(a.force, a.alpha, a.dens, B.n, n2, mf2, mu - din2, a.alpha_burst, a.growth, n) : 0;
        const bool cont = n2 > 0 && dir2 == TSMV_DIR_PUSH_CSC && mx2 <= LIST_MAXW && n2 <= SOLO_QS &&
                          ss.W <= SOLO_ITEMS && level < a.max_levels;
        SOLO_T(3);
        if (!cont) {
#ifdef TSMV_SOLO_PROF
            if (tid == 0 && nlev > 100)
                printf("solo %lld levels: cycles/level loads %lld atomics %lld records %lld decide %lld tail %lld\n",
                       nlev, pc[0] / nlev, pc[1] / nlev, pc[2] / nlev, pc[3] / nlev, pc[4] / nlev);
#endif
            // leave frontier `level` in the global list + its slot, slot level+1 zeroed
            fprev = n;
            int *Qg = (level & 1) ? a.bq1 : a.bq0;
            for (long long i = tid; i < min(n2, (long long)SOLO_QS); i += BFB) Qg[i] = sb.nq[i];
            if (tid == 0) {
                long long *sl = a.lslots + (level % 3) * 4, *sn = a.lslots + ((level + 1) % 3) * 4;
                sl[0] = n2;
                sl[1] = mf2;
                sl[2] = din2;
                sl[3] = mx2;
                sn[0] = sn[1] = sn[2] = sn[3] = 0;
            }
            __syncthreads();
            return;
        }
        mu -= din2;
        reached += n2;
        edges += mf2;
        if (tid == 0 && level < TSMV_MAX_LEVELS) {
            a.dir_out[level] = dir2;
            a.front_out[level] = n2;
            a.tlv_out[level] = globaltimer_ns();
        }
        n = n2;
#ifdef TSMV_SOLO_PROF
        ++nlev;
#endif
        SOLO_T(4);
    }
}

#ifndef TSMV_BFS_MINB
#define TSMV_BFS_MINB 1
#endif
template <int NT>
__global__ void __launch_bounds__(BFB, TSMV_BFS_MINB) k_bfs_fused(BfsFusedArgs a) {
    using word_t = typename Tr<NT>::word_t;
    constexpr int NWP = BFB / 32;
    __shared__ long long s_scan[16][NWP];
    __shared__ long long s_tot[8], s_pre[8];
    __shared__ long long win_all[NWP][CHUNK + 1];
    const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
    const int G = gridDim.x, b = blockIdx.x;
    const long long gtid = (long long)b * BFB + tid, gthreads = (long long)G * BFB;
    const long long gwarp = gtid >> 5, gwarps = gthreads >> 5;
    unsigned long long target = a.bar_base;
    BfsView B = a.B;
    uint32_t *Fa = B.F, *Fb = B.Fn;

    __shared__ ListShared sh;
    __shared__ long long s_hv[HVQ][3];  // chunk-map runs too long for one thread (hub columns)
    __shared__ int s_nhv;
    __shared__ SoloBuf s_solo_buf;
    __shared__ SoloShared s_solo;
    unsigned long long solo_n = 0;  // solo episodes of this launch (same in every CTA)
    int mode_list = a.use_list && !a.resume;

    // ---- init: V = padding bits + source, F0 = {source} (scan mode) or the
    // list {source} (list mode), F1 = 0, levels
    for (long long w = gtid; w < (a.resume ? 0 : a.NW); w += gthreads) {
        const long long v0 = w * 32;
        uint32_t pad = 0;
        if (v0 + 32 > B.n) pad = (v0 >= B.n) ? 0xffffffffu : (0xffffffffu << (B.n - v0));
        const uint32_t s = (a.source >= v0 && a.source < v0 + 32) ? (1u << (a.source - v0)) : 0u;
        B.V[w] = pad | s;
        Fa[w] = mode_list ? 0u : s;
        Fb[w] = 0;
    }
    if (!a.resume)
        for (long long v = gtid; v < B.m_local; v += gthreads) B.levels[v] = (v == a.source) ? 0 : -1;
    if (tid == 0) {
        sh.qn = 0;
        sh.maxw = 0;
        sh.mf = 0;
        sh.din = 0;
    }
    // L2 warm-up (fire and forget: the first levels do not wait for it)
    for (int r = 0; r < a.pf_n; ++r) {
        const char *base = (const char *)a.pf_p[r];
        const long long nb = a.pf_b[r] & ~15LL;
        for (long long ch = gtid; ch * PF_CHUNK < nb; ch += gthreads) {
            const unsigned sz = (unsigned)min(PF_CHUNK, nb - ch * PF_CHUNK);
            asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(base + ch * PF_CHUNK), "r"(sz) : "memory");
        }
    }
    if (mode_list && b == 0 && tid == 0) {
        a.bq0[0] = (int)a.source;
        a.lslots[0] = 1;
        a.lslots[1] = a.outdeg[a.source];
        a.lslots[2] = a.indeg[a.source];
        a.lslots[3] = a.lwork[a.source];
        for (int i = 4; i < 12; ++i) a.lslots[i] = 0;
    }
    grid_sync(&a.cnt->bar, target);

    long long mu = a.resume ? a.mu0 : a.nnz, reached = a.reached0, edges = a.edges0;
    int stopped = 0;
    bool relist = false;  // a scan level converted back to a list level (counted already)
    const long long S = (a.nseg + G - 1) / G;                 // segments per CTA
    const long long js0 = (long long)b * S, js1 = min(a.nseg, js0 + S);
    const long long per = (S + BFB - 1) / BFB;
    const long long tj0 = min(js1, js0 + tid * per), tj1 = min(js1, tj0 + per);
    int level = (int)a.level0;
    long long fprev = a.fprev0;  // |F| of the previous level (R9')
    unsigned long long t_s1 = 0, t_s2 = 0, t_e = 0, tq = b == 0 && tid == 0 ? globaltimer_ns() : 0;
    bool redo = false;  // scan pass over a level already counted in list mode
    for (; level < a.max_levels; ++level) {
        B.F = Fa;
        B.Fn = Fb;
        B.level = level;
        if (mode_list) {
            // ---- list level: counters of this level from its slot
            const long long *sl = a.lslots + (level % 3) * 4;
            const long long fsize = __ldcg(&sl[0]), mf = __ldcg(&sl[1]), din = __ldcg(&sl[2]),
                            maxw = __ldcg(&sl[3]);
            if (!relist) mu -= din;
            if (fsize == 0) break;
            if (!relist) {
                reached += fsize;
                edges += mf;
            }
            const int dir = choose_dir_dev(a.force, a.alpha, a.dens, B.n, fsize, mf, mu, a.alpha_burst, a.growth,
                                           fprev);
            if (b == 0 && tid == 0 && level < TSMV_MAX_LEVELS && !relist) {
                a.dir_out[level] = dir;
                a.front_out[level] = fsize;
                a.tlv_out[level] = globaltimer_ns();
            }
            relist = false;
            const int *Qc = (level & 1) ? a.bq1 : a.bq0;
            if (dir != TSMV_DIR_PUSH_CSC || maxw > LIST_MAXW) {
                // hand the level to the scan form: list -> frontier bitmap Fa
                for (long long i = gtid; i < fsize; i += gthreads) {
                    const long long v = __ldcg(&Qc[i]);
                    atomicOr(&Fa[v >> 5], 1u << (v & 31));
                }
                grid_sync(&a.cnt->bar, target);
                mode_list = 0;
                redo = true;
                --level;  // the loop increment brings it back
                continue;
            }
            int *Qn = (level & 1) ? a.bq0 : a.bq1;
            long long *slot_n = a.lslots + ((level + 1) % 3) * 4;
            int G = 1;
            while (G < maxw && G < 32) G <<= 1;
            if (a.use_solo && fsize <= SOLO_QS && fsize * maxw <= SOLO_ITEMS) {
                // small frontier: CTA 0 runs the next levels alone (solo_levels)
                ++solo_n;
                if (b == 0) {
                    fprev = fsize;
                    solo_levels<NT>(a, B, level, mu, reached, edges, fsize, fprev, s_solo_buf, s_solo, tid);
                    if (tid == 0) {
                        a.lslots[17] = level;
                        a.lslots[18] = mu;
                        a.lslots[19] = reached;
                        a.lslots[20] = edges;
                        a.lslots[21] = fprev;
                        __threadfence();
                        atomicExch((unsigned long long *)&a.lslots[16], solo_n);
                    }
                    __syncthreads();
                } else {
                    if (tid == 0) {
                        while (ld_acquire_u64((const unsigned long long *)&a.lslots[16]) < solo_n) __nanosleep(256);
                        __threadfence();
                    }
                    __syncthreads();
                    level = (int)__ldcg(&a.lslots[17]);
                    mu = __ldcg(&a.lslots[18]);
                    reached = __ldcg(&a.lslots[19]);
                    edges = __ldcg(&a.lslots[20]);
                    fprev = __ldcg(&a.lslots[21]);
                }
                if (b == 0 && tid == 0) {
                    const unsigned long long t = globaltimer_ns();
                    t_e += t - tq;
                    tq = t;
                }
                --level;  // the loop increment brings it back
                continue;
            }
#ifdef TSMV_LIST_PROF
            unsigned long long tl0 = 0, tl1 = 0, tl2 = 0;
            if (b == 0 && tid == 0) tl0 = globaltimer_ns();
#endif
            fprev = fsize;
            list_level<NT>(a, B, Qc, fsize, G, gtid, gthreads, sh, Qn, slot_n);
#ifdef TSMV_LIST_PROF
            __syncthreads();
            if (b == 0 && tid == 0) tl1 = globaltimer_ns();
            if (tid == 0) atomicMax((unsigned long long *)&a.lslots[12 + (level % 3)], globaltimer_ns());
#endif
            if (b == 0 && tid == 0) {
                long long *sz = a.lslots + ((level + 2) % 3) * 4;
                sz[0] = sz[1] = sz[2] = sz[3] = 0;
            }
            list_flush(a, sh, Qn, slot_n, tid, lane);
            __syncthreads();
            if (tid == 0) {
                sh.qn = 0;
                sh.maxw = 0;
                sh.mf = 0;
                sh.din = 0;
            }
#ifdef TSMV_LIST_PROF
            if (b == 0 && tid == 0) tl2 = globaltimer_ns();
#endif
            grid_sync(&a.cnt->bar, target);
            if (b == 0 && tid == 0) {
                const unsigned long long t = globaltimer_ns();
                t_e += t - tq;
                tq = t;
#ifdef TSMV_LIST_PROF
                // t_s1: CTA 0 expansion, t_s2: slowest CTA's expansion end - CTA 0 start,
                // lslots[15]: CTA 0 flush
                t_s1 += tl1 - tl0;
                unsigned long long *cell = (unsigned long long *)&a.lslots[12 + (level % 3)];
                t_s2 += __ldcg(cell) - tl0;
                a.lslots[15] += (long long)(tl2 - tl1);
                *(unsigned long long *)&a.lslots[12 + ((level + 2) % 3)] = 0;
#endif
            }
            continue;
        }
        // ---- S: count this thread's segments, clear the consumed bitmap Fb
        if (a.use_list && b == 0 && tid == 0) {
            // slots a conversion back to list levels (below) would use: this level's
            // max-work cell and the next level's counters
            a.lslots[(level % 3) * 4 + 3] = 0;
            long long *sz = a.lslots + ((level + 1) % 3) * 4;
            sz[0] = sz[1] = sz[2] = sz[3] = 0;
        }
        long long v[8] = {0, 0, 0, 0, 0, 0, 0, 0};
        for (long long J = tj0; J < tj1; ++J) {
            seg_counts<NT>(a, Fa, J, v);
            if constexpr (NT == 16) {
                Fb[J >> 1] = 0u;  // both halves of the word are in this slice or cleared twice
            } else if constexpr (NT == 32) {
                Fb[J] = 0u;
            } else {
                Fb[2 * J] = 0u;
                Fb[2 * J + 1] = 0u;
            }
        }
        long long ex[8], tot[8];
        block_scan<8, BFB>(v, ex, tot, s_scan);
        if (tid < 8) a.partials[b * 8 + tid] = tot[tid];
        if (b == 0 && tid == 0) a.cnt->chunk_next = 0;
        grid_sync(&a.cnt->bar, target);
        if (b == 0 && tid == 0) {
            const unsigned long long t = globaltimer_ns();
            t_s1 += t - tq;
            tq = t;
        }
        // totals and this CTA's prefix of the 7 counts: every thread loads its
        // (CTA, count) cells at once (one round trip, not one per 32 CTAs), lanes
        // l, l+8, l+16, l+24 of a warp hold the same count: two shuffles, then one
        // shared-memory add per warp and count
        if (tid < 8) {
            s_pre[tid] = 0;
            s_tot[tid] = 0;
        }
        __syncthreads();
        {
            constexpr int PQ = (MAXBG * 8 + BFB - 1) / BFB;
            long long xa[PQ], xp[PQ];
#pragma unroll
            for (int k = 0; k < PQ; ++k) {
                const int q = tid + k * BFB;
                const long long x = q < G * 8 && (q & 7) < 7 ? __ldcg(&a.partials[q]) : 0;
                xa[k] = x;
                xp[k] = (q >> 3) < b ? x : 0;
            }
            long long ta = 0, tp = 0;
#pragma unroll
            for (int k = 0; k < PQ; ++k) {
                ta += xa[k];
                tp += xp[k];
            }
            // q & 7 == tid & 7 for every k (BFB is a multiple of 8)
            ta += __shfl_xor_sync(0xffffffffu, ta, 8);
            tp += __shfl_xor_sync(0xffffffffu, tp, 8);
            ta += __shfl_xor_sync(0xffffffffu, ta, 16);
            tp += __shfl_xor_sync(0xffffffffu, tp, 16);
            if (lane < 7) {
                if (ta) atomicAdd((unsigned long long *)&s_tot[lane], (unsigned long long)ta);
                if (tp) atomicAdd((unsigned long long *)&s_pre[lane], (unsigned long long)tp);
            }
        }
        __syncthreads();
        const long long fsize = s_tot[4], mf = s_tot[5];
        if (!redo) mu -= s_tot[6];
        if (fsize == 0) break;
        if (!redo) {
            reached += fsize;
            edges += mf;
        }
        redo = false;
        const int dir = choose_dir_dev(a.force, a.alpha, a.dens, B.n, fsize, mf, mu, a.alpha_burst, a.growth, fprev);
        if (b == 0 && tid == 0 && level < TSMV_MAX_LEVELS) {
            a.dir_out[level] = dir;
            a.front_out[level] = fsize;
            a.tlv_out[level] = globaltimer_ns();
        }
        // Dense pull levels go back to the host's high-occupancy kernels; pull
        // levels with few unvisited edges (m_u <= 16 per thread of this grid, or
        // m_u < nnz / 4: late R-MAT levels, small graphs, the tail of a
        // high-diameter traversal) run here with the wide row-tile test
        // (r2) and late pull levels that are still large in absolute terms (> wide_cap
        // unvisited edges: s26) go to the host kernels too, whose occupancy the
        // latency-bound wide pull needs more than it needs the saved round trip
        if (dir == TSMV_DIR_PULL_CSC && a.stop_on_pull && mu > 16 * gthreads &&
            (!a.wide_in_kernel || mu * 4 >= a.nnz || mu > a.wide_cap)) {
            stopped = 1;  // uniform across CTAs: same totals, same decision
            fprev = fsize;  // handed to the host: |F| of the level it expands
            break;
        }
        if (a.use_list && dir == TSMV_DIR_PUSH_CSC && fsize * 64 <= B.n && !a.no_relist) {
            // a small Push-CSC frontier after scan levels (the tail of an R-MAT
            // traversal): the bitmap frontier becomes this level's list (positions
            // from the count phase's prefix, no atomics) and the level runs as a
            // list level, so the following small levels are list / solo levels
            // (one grid barrier, or none) instead of scans of the whole bitmap
            int *Qw = (level & 1) ? a.bq1 : a.bq0;
            long long *sl = a.lslots + (level % 3) * 4;
            long long pos = s_pre[4] + ex[4];
            int mx = 0;
            for (long long J = tj0; J < tj1; ++J) {
                word_t bits = seg_bits<NT>(Fa, J);
                while (bits) {
                    const int r = ffs_w(bits);
                    bits &= bits - 1;
                    const long long u = J * NT + r;
                    Qw[pos++] = (int)u;
                    mx = max(mx, a.lwork[u]);
                }
            }
#pragma unroll
            for (int o = 16; o > 0; o >>= 1) mx = max(mx, __shfl_xor_sync(0xffffffffu, mx, o));
            if (lane == 0 && mx) atomicMax(&sl[3], (long long)mx);
            if (b == 0 && tid == 0) {
                sl[0] = fsize;
                sl[1] = mf;
                sl[2] = s_tot[6];
            }
            grid_sync(&a.cnt->bar, target);
            if (__ldcg(&sl[3]) <= LIST_MAXW) {
                // the list level does not read the bitmaps: clear this level's
                // frontier words (read by every thread before the barrier above)
                for (long long J = tj0; J < tj1; ++J) {
                    if constexpr (NT == 16) Fa[J >> 1] = 0u;
                    else if constexpr (NT == 32) Fa[J] = 0u;
                    else {
                        Fa[2 * J] = 0u;
                        Fa[2 * J + 1] = 0u;
                    }
                }
                mode_list = 1;
                relist = true;
                --level;  // the loop increment brings it back
                continue;
            }
        }
        fprev = fsize;
        // lists (Push-CSC needs both, Push-CSR the side list; pull none)
        if (dir != TSMV_DIR_PULL_CSC) {
            if (tid == 0) s_nhv = 0;
            __syncthreads();
            long long oLt = s_pre[0] + ex[0], oWt = s_pre[1] + ex[1];
            long long oLs = s_pre[2] + ex[2], oWs = s_pre[3] + ex[3];
            for (long long J = tj0; J < tj1; ++J) {
                const word_t bits = seg_bits<NT>(Fa, J);
                if (!bits) continue;
                const long long wt = a.P.ptr[J + 1] - a.P.ptr[J];
                if (wt > 0) {
                    a.Lv.Lt_seg[oLt] = J;
                    a.Lv.Lt_mask[oLt] = (unsigned long long)bits;
                    a.Lv.Lt_tbeg[oLt] = a.P.ptr[J];
                    a.Lv.Lt_wpre[oLt] = oWt;
                    put_chunks_q(a.Lv.Ct, oWt, wt, (int)oLt, 0, s_hv, &s_nhv);
                    ++oLt;
                    oWt += wt;
                }
                word_t bb = bits;
                while (bb) {
                    const int r = ffs_w(bb);
                    bb &= bb - 1;
                    const long long u = J * NT + r;
                    const long long ws = a.P.sptr[u + 1] - a.P.sptr[u];
                    if (ws > 0) {
                        a.Lv.Ls_beg[oLs] = a.P.sptr[u];
                        a.Lv.Ls_wpre[oLs] = oWs;
                        put_chunks_q(a.Lv.Cs, oWs, ws, (int)oLs, 1, s_hv, &s_nhv);
                        ++oLs;
                        oWs += ws;
                    }
                }
            }
            if (b == G - 1 && tid == 0) {
                a.Lv.Lt_wpre[s_tot[0]] = s_tot[1];
                a.Lv.Ls_wpre[s_tot[2]] = s_tot[3];
            }
            __syncthreads();
            // queued long runs, a warp each
            for (int h = wid; h < min(s_nhv, HVQ); h += NWP) {
                int *C = s_hv[h][2] >> 32 ? a.Lv.Cs : a.Lv.Ct;
                const int entry = (int)(s_hv[h][2] & 0xffffffffll);
                for (long long ch = s_hv[h][0] + lane; ch < s_hv[h][1]; ch += 32) C[ch] = entry;
            }
        }
        grid_sync(&a.cnt->bar, target);
        if (b == 0 && tid == 0) {
            const unsigned long long t = globaltimer_ns();
            t_s2 += t - tq;
            tq = t;
        }

        // a heavy Push-CSC level (bulk mode, >= bulk_stop_min items: R-MAT s26's hub
        // levels, ~90 M edges) is handed to the host's high-occupancy k_push /
        // k_bulk_fix over the lists just built (this kernel runs 16 warps per SM:
        // 2.1 ms for that level against 1.0 ms there); the kernel resumes after it
        if (a.stop_on_bulk && dir == TSMV_DIR_PUSH_CSC && a.bulk_push && (s_tot[1] + s_tot[3]) * 8 > B.n &&
            s_tot[1] + s_tot[3] >= a.bulk_stop_min) {
            if (b == 0 && tid == 0) {
                a.cnt->nLt = s_tot[0];
                a.cnt->Wt = s_tot[1];
                a.cnt->nLs = s_tot[2];
                a.cnt->Ws = s_tot[3];
                a.cnt->nCt = (s_tot[1] + CHUNK - 1) >> CHUNK_LOG;
                a.cnt->nCs = (s_tot[3] + CHUNK - 1) >> CHUNK_LOG;
            }
            stopped = 2;  // uniform across CTAs
            break;
        }
        // ---- E: expand
        bool bulk = false;
        if (dir == TSMV_DIR_PULL_CSC) {
            for (long long I0 = gwarp * 32; I0 < a.nTR_local; I0 += gwarps * 32)
                pull_rowtiles32<NT>(a.Q, B, I0, a.nTR_local, lane);
            for (long long w = gtid; w < (B.m_local + 31) / 32; w += gthreads) pull_side_word<NT>(a.Q, B, w);
        } else {
            if (dir == TSMV_DIR_PUSH_CSR)
                for (long long t = gtid; t < a.Q.T; t += gthreads) push_csr_item<NT>(a.Q, B, t);
            const long long nLt = s_tot[0], Wt = s_tot[1], nLs = s_tot[2], Ws = s_tot[3];
            const long long nCt = dir == TSMV_DIR_PUSH_CSC ? (Wt + CHUNK - 1) >> CHUNK_LOG : 0;
            const long long nCs = (Ws + CHUNK - 1) >> CHUNK_LOG;
            // heavy Push-CSC level (push items > n / 8): bulk mode, reductions into Fn
            // then one pass over the words (below)
            bulk = a.bulk_push && dir == TSMV_DIR_PUSH_CSC && (Wt + Ws) * 8 > B.n;
            long long *win = win_all[wid];
            unsigned ch = (unsigned)gwarp;
            while (true) {
                unsigned nx = 0;
                if (lane == 0 && ch < nCt + nCs) nx = (unsigned)gwarps + atomicAdd(&a.cnt->chunk_next, 1u);
                if (ch < nCt) {
                    const long long s0 = __ldcg(&a.Lv.Ct[ch]);
                    const long long base = (long long)ch << CHUNK_LOG;
                    load_window(win, a.Lv.Lt_wpre, s0, nLt, lane);
#pragma unroll
                    for (int u = 0; u < CHUNK / 32; ++u) {
                        const long long i = base + lane + 32 * u;
                        if (i < Wt) {
                            const int q = window_find(win, i);
                            const long long s = s0 + q;
                            push_tile_item<NT>(a.P, B, __ldcg(&a.Lv.Lt_tbeg[s]) + (i - win[q]),
                                               (word_t)__ldcg(&a.Lv.Lt_mask[s]), bulk);
                        }
                    }
                } else if (ch < nCt + nCs) {
                    const long long c2 = (long long)ch - nCt;
                    const long long s0 = __ldcg(&a.Lv.Cs[c2]);
                    const long long base = c2 << CHUNK_LOG;
                    load_window(win, a.Lv.Ls_wpre, s0, nLs, lane);
#pragma unroll
                    for (int u = 0; u < CHUNK / 32; ++u) {
                        const long long i = base + lane + 32 * u;
                        if (i < Ws) {
                            const int q = window_find(win, i);
                            push_side_item<NT>(a.P, B, __ldcg(&a.Lv.Ls_beg[s0 + q]) + (i - win[q]), bulk);
                        }
                    }
                } else {
                    break;
                }
                __syncwarp();
                ch = __shfl_sync(0xffffffffu, nx, 0);
            }
        }
        grid_sync(&a.cnt->bar, target);
        if (bulk) {
            // new = Fn & ~V over all words (every reduction of the level has landed)
            for (long long w = gtid; w < a.NW; w += gthreads) {
                const uint32_t f = Fb[w];
                if (!f) continue;
                const uint32_t v = B.V[w];
                const uint32_t nw = f & ~v;
                Fb[w] = nw;
                if (nw) {
                    B.V[w] = v | nw;
                    uint32_t bb = nw;
                    while (bb) {
                        const int r = __ffs(bb) - 1;
                        bb &= bb - 1;
                        B.levels[w * 32 + r] = level + 1;
                    }
                }
            }
            grid_sync(&a.cnt->bar, target);
        }
        if (b == 0 && tid == 0) {
            const unsigned long long t = globaltimer_ns();
            t_e += t - tq;
            tq = t;
        }
        uint32_t *tmp = Fa;
        Fa = Fb;
        Fb = tmp;
    }
    if (b == 0 && tid == 0) {
        a.hm->fsize = level;  // levels finished (or the level stopped at)
        a.hm->reached = reached;
        a.hm->edges = edges;
        a.hm->mf = mu;
        a.hm->din = stopped;
        a.hm->nCt = fprev;  // |F| of the last level decided (the stopped one when stopped)
        a.hm->nLt = (Fa == a.B.F) ? 0 : 1;  // which bitmap holds the current frontier
        a.hm->Wt = (long long)t_s1;  // phase times (ns, CTA 0): count, lists, expand
        a.hm->nLs = (long long)t_s2;
        a.hm->Ws = (long long)t_e;
        a.hm->bfs_bars = target - a.bar_base;  // = G x barriers passed
    }
}

// lwork[u] = tiles of u's tile column + u's side nonzeros (push work of u in a list level)
__global__ void k_lwork(const long long *__restrict__ ptr, const long long *__restrict__ sptr, int lognt,
                        long long n, int *__restrict__ lwork) {
    for (long long u = blockIdx.x * (long long)blockDim.x + threadIdx.x; u < n;
         u += (long long)gridDim.x * blockDim.x) {
        const long long J = u >> lognt;
        const long long w = (ptr[J + 1] - ptr[J]) + (sptr[u + 1] - sptr[u]);
        lwork[u] = (int)min(w, (long long)INT_MAX);
    }
}

}  // namespace

void bfs_list_init(tsmv_ctx *c, cudaStream_t st) {
    c->lwork.alloc(std::max<int64_t>(c->n, 1) * 4);
    c->bq0.alloc(std::max<int64_t>(c->n, 1) * 4);
    c->bq1.alloc(std::max<int64_t>(c->n, 1) * 4);
    c->lslots.alloc(24 * 8);
    TSMV_CUDA(cudaMemsetAsync(c->lslots.p, 0, c->lslots.bytes, st));
    const long long n = c->n;
    const int grid = (int)std::max<long long>(1, std::min<long long>((n + 255) / 256, 148LL * 16));
    k_lwork<<<grid, 256, 0, st>>>(c->P.ptr.as<long long>(), c->P.sptr.as<long long>(), c->lognt, n,
                                  c->lwork.as<int>());
    TSMV_CUDA(cudaGetLastError());
}

int bfs_fused_occupancy(int nt) {
    int bps = 0;
    cudaError_t e = cudaSuccess;
    if (nt == 16) e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&bps, k_bfs_fused<16>, BFB, 0);
    else if (nt == 32) e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&bps, k_bfs_fused<32>, BFB, 0);
    else e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&bps, k_bfs_fused<64>, BFB, 0);
    if (e != cudaSuccess) {
        cudaGetLastError();
        bps = 0;
    }
    return bps;
}

// in-kernel wide pull only while m_u <= 16 edges per thread of the persistent grid
// (measured: R-MAT s22 / s26); resume = the host's test for handing a
// late pull level back to the fused kernel, which also needs the kernel's bitmap
// scan to be short: <= 4 nt-segments per thread (s22 yes, s26 no)
long long bfs_wide_cap(const tsmv_ctx *c, bool resume) {
    const char *e = getenv(resume ? "TSMV_BFS_RESUME_CAP" : "TSMV_BFS_WIDE_CAP");
    const double mult = e ? atof(e) : 16.0;
    const long long threads = (long long)c->bfs_blocks * BFB;
    if (resume && !e && c->nTC > 4 * threads) return -1;
    return (long long)(mult * (double)threads);
}

// Launch the fused kernel from `level0` (resume) on bitmaps (Fa, Fb).  Returns
// true if it stopped before a Pull-CSC level.
bool bfs_fused_launch(tsmv_ctx *c, long long source, cudaStream_t st, bool resume, long long level0, uint32_t *Fa,
                      uint32_t *Fb, long long mu, long long reached, long long edges, bool stop_on_pull,
                      long long max_levels, long long &level_out, long long &mu_out, long long &reached_out,
                      long long &edges_out, int &cur_out, long long fprev0, long long &fprev_out) {
    BfsFusedArgs a;
    a.P = bfs_tiles(c->P);
    a.Q = bfs_tiles(*c->Q);
    a.B.V = c->V.as<uint32_t>();
    a.B.F = Fa;
    a.B.Fn = Fb;
    a.B.levels = c->levels_dev;
    a.B.row_begin = 0;
    a.B.m_local = c->m;
    a.B.n = c->n;
    a.B.level = 0;
    a.outdeg = c->outdeg.as<int>();
    a.indeg = c->indeg.as<int>();
    a.Lv = lists_view(c);
    a.partials = c->partials.as<long long>();
    a.cnt = c->counters.as<Counters>();
    a.hm = c->hcnt_dev;
    a.dir_out = c->bfs_dirs.as<int>();
    a.front_out = c->bfs_front.as<long long>();
    a.tlv_out = c->bfs_tlv.as<unsigned long long>();
    a.source = source;
    a.nnz = c->nnz;
    a.nseg = c->nTC;
    a.NW = (long long)(c->V.bytes / 4);
    a.nTR_local = (c->m + c->nt - 1) / c->nt;
    a.max_levels = max_levels;
    a.alpha = c->opt.pull_alpha;
    a.dens = c->opt.push_csr_density;
    a.force = c->opt.force_dir;
    a.alpha_burst = c->opt.pull_alpha_burst;
    a.growth = c->opt.burst_growth;
    a.fprev0 = fprev0;
    a.bar_base = c->bar_base;
    a.resume = resume ? 1 : 0;
    a.stop_on_pull = stop_on_pull ? 1 : 0;
    a.level0 = level0;
    a.mu0 = mu;
    a.reached0 = reached;
    a.edges0 = edges;
    a.lwork = c->lwork.as<int>();
    a.bq0 = c->bq0.as<int>();
    a.bq1 = c->bq1.as<int>();
    a.lslots = c->lslots.as<long long>();
    a.use_list = (c->lwork.p != nullptr && !getenv("TSMV_BFS_NO_LIST")) ? 1 : 0;
    // solo records hold 32-bit tile / side starts
    a.no_relist = getenv("TSMV_BFS_NO_RELIST") ? 1 : 0;
    a.stop_on_bulk = (stop_on_pull && !(getenv("TSMV_BFS_BULK_HOST") && atoi(getenv("TSMV_BFS_BULK_HOST")) == 0)) ? 1 : 0;
    a.bulk_stop_min = getenv("TSMV_BFS_BULK_HOST_MIN") ? atoll(getenv("TSMV_BFS_BULK_HOST_MIN")) : (4ll << 20);
    a.use_solo = a.use_list && !getenv("TSMV_BFS_NO_SOLO") && c->P.T < (1LL << 32) && c->P.side_nnz < (1LL << 32)
                     ? 1 : 0;
    a.wide_in_kernel = getenv("TSMV_BFS_HOST_WIDE") ? 0 : 1;
    a.wide_cap = bfs_wide_cap(c, false);
    a.bulk_push = getenv("TSMV_BFS_NO_BULK") ? 0 : 1;
    a.qcap = getenv("TSMV_BFS_QCAP") ? std::max(1, std::min(QCAP, atoi(getenv("TSMV_BFS_QCAP")))) : QCAP;
    if (a.use_solo) TSMV_CUDA(cudaMemsetAsync(c->lslots.as<long long>() + 16, 0, 8, st));  // release flag
    a.pf_n = 0;
    {
        const TileSet &P = c->P;
        const DevBuf *bufs[8] = {&P.ptr, &P.sptr, &P.planes, &P.trow, &P.srow, &c->outdeg, &c->indeg, &c->lwork};
        long long tot = 0;
        for (const DevBuf *d : bufs) tot += (long long)d->bytes;
        int l2 = 0;
        cudaDeviceGetAttribute(&l2, cudaDevAttrL2CacheSize, c->device);
        const char *e = getenv("TSMV_BFS_L2PF");
        const bool on = e ? atoi(e) != 0 : (!resume && a.use_list && tot <= (long long)l2 / 2);
        if (on)
            for (const DevBuf *d : bufs)
                if (d->p && d->bytes >= 16) {
                    a.pf_p[a.pf_n] = d->p;
                    a.pf_b[a.pf_n] = (long long)d->bytes;
                    ++a.pf_n;
                }
    }
    void *args[] = {&a};
    void *f = c->nt == 16 ? (void *)k_bfs_fused<16> : c->nt == 32 ? (void *)k_bfs_fused<32> : (void *)k_bfs_fused<64>;
    const int G = std::min(c->bfs_blocks, MAXBG);
    TSMV_CUDA(cudaLaunchCooperativeKernel(f, dim3(G), dim3(BFB), args, 0, st));
    TSMV_CUDA(cudaStreamSynchronize(st));
    volatile Counters *h = c->hcnt;
    const long long L = h->fsize;
    const bool stopped = h->din != 0;
    c->bfs_stop_kind = (int)h->din;  // 1: a pull level, 2: a heavy bulk push level (lists built)
    level_out = L;
    reached_out = h->reached;
    edges_out = h->edges;
    mu_out = h->mf;
    cur_out = (int)h->nLt;
    fprev_out = h->nCt;
    c->bar_base += h->bfs_bars;
    return stopped;
}

}  // namespace tsmv
