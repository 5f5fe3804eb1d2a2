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
#include "bfs_dev.cuh"

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

// per-level device time (tsmv_bfs_stats::level_ms): %globaltimer of a level the
// host runs itself, and of the end of the traversal
__global__ void k_stamp(unsigned long long *t) { *t = globaltimer_ns(); }
// per-level record of a host-decided level: direction, frontier size, time stamp
// (one launch on the stream instead of two synchronous copies and a launch)
__global__ void k_level_rec(int *dirs, long long *front, unsigned long long *tlv, int dir, long long f) {
    *dirs = dir;
    *front = f;
    *tlv = globaltimer_ns();
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

// One nt-segment J of the frontier bitmap F: q.v[0..3] = list terms (segment
// has tile work, its tile work, side columns with entries, their side work),
// with `full` also q.v[4..6] = |F| bits, m_f, sum of in-degrees of local rows.
template <int NT>
__device__ __forceinline__ typename Tr<NT>::word_t
scan_seg(const uint32_t *__restrict__ F, long long J, const long long *__restrict__ tptr,
         const long long *__restrict__ sptr, const int *__restrict__ outdeg, const int *__restrict__ indeg,
         long long row_begin, long long m_local, bool full, Oct &q, long long &wt) {
    using word_t = typename Tr<NT>::word_t;
#pragma unroll
    for (int i = 0; i < 8; ++i) q.v[i] = 0;
    wt = 0;
    const word_t bits = seg_bits<NT>(F, J);
    if (!bits) return bits;
    wt = tptr[J + 1] - tptr[J];
    q.v[0] = wt > 0;
    q.v[1] = wt;
    if constexpr (NT == 16) {
        // the segment's 16 out-degrees, in-degrees and 17 side starts are
        // contiguous: 4 + 4 + 9 independent 16-byte loads, one latency
        const long long v0 = J * 16;
        const longlong2 *sp2 = reinterpret_cast<const longlong2 *>(sptr + v0);
        long long sp[18];
#pragma unroll
        for (int i = 0; i < 8; ++i) {
            const longlong2 t = __ldg(sp2 + i);
            sp[2 * i] = t.x, sp[2 * i + 1] = t.y;
        }
        sp[16] = __ldg(sptr + v0 + 16);
        int od[16], id[16];
#pragma unroll
        for (int r = 0; r < 16; ++r) od[r] = id[r] = 0;
        if (full) {
            q.v[4] = popc_w(bits);
            const int4 *od4 = reinterpret_cast<const int4 *>(outdeg + v0);
#pragma unroll
            for (int i = 0; i < 4; ++i) {
                const int4 t = __ldg(od4 + i);
                od[4 * i] = t.x, od[4 * i + 1] = t.y, od[4 * i + 2] = t.z, od[4 * i + 3] = t.w;
            }
            const long long lv0 = v0 - row_begin;
            if (lv0 >= 0 && lv0 + 16 <= m_local) {
                const int4 *id4 = reinterpret_cast<const int4 *>(indeg + lv0);
#pragma unroll
                for (int i = 0; i < 4; ++i) {
                    const int4 t = __ldg(id4 + i);
                    id[4 * i] = t.x, id[4 * i + 1] = t.y, id[4 * i + 2] = t.z, id[4 * i + 3] = t.w;
                }
            } else {
#pragma unroll
                for (int r = 0; r < 16; ++r)
                    id[r] = (lv0 + r >= 0 && lv0 + r < m_local) ? __ldg(indeg + lv0 + r) : 0;
            }
        }
#pragma unroll
        for (int r = 0; r < 16; ++r) {
            if ((bits >> r) & 1u) {
                const long long ws = sp[r + 1] - sp[r];
                q.v[2] += ws > 0;
                q.v[3] += ws;
                q.v[5] += od[r];
                q.v[6] += id[r];
            }
        }
    } else {
        word_t b = bits;
        while (b) {
            int r = ffs_w(b);
            b &= b - 1;
            long long v = J * NT + r;
            long long ws = sptr[v + 1] - sptr[v];
            q.v[2] += ws > 0;
            q.v[3] += ws;
            if (full) {
                q.v[5] += outdeg[v];
                long long lv = v - row_begin;
                if (lv >= 0 && lv < m_local) q.v[6] += indeg[lv];
            }
        }
        if (full) q.v[4] = popc_w(bits);
    }
    return bits;
}

// Frontier scan over the nseg nt-segments of the (global) frontier bitmap F.
// One wave of blocks, each owning a contiguous range of `tpb` super-tiles; a
// super-tile is SCAN_BLOCK threads x SPT = 128/nt consecutive segments, one
// 16-byte load of F per thread, so an empty stretch of the frontier costs one
// coalesced read (r2: a block per 256 segments made a 4096-block look-back chain
// at scale 24 -- 144 us for a one-vertex frontier):
//   pass 1: per-segment terms of the whole range, block aggregate, clear Fclear;
//   (statistics only: block reduction + atomics, the last block publishes)
//   look-back for the range's exclusive prefix;
//   pass 2: super-tiles with a frontier bit again, block-exclusive-scan of the
//           four list terms + running offset, write the tile / side lists and
//           chunk starts, each thread its SPT segments in order.
template <int NT>
__device__ __forceinline__ uint4 ld_f4(const uint32_t *__restrict__ F, long long w, long long nwpad) {
    return w + 4 <= nwpad ? __ldg(reinterpret_cast<const uint4 *>(F + w)) : make_uint4(0u, 0u, 0u, 0u);
}

template <int NT>
__global__ void __launch_bounds__(SCAN_BLOCK)
k_fscan(const uint32_t *__restrict__ F, uint32_t *__restrict__ Fclear, long long nseg, long long tpb,
        long long nwpad, const long long *__restrict__ tptr, const long long *__restrict__ sptr,
        const int *__restrict__ outdeg, const int *__restrict__ indeg, long long row_begin, long long m_local,
        ListsView Lv, Counters *__restrict__ cnt, Counters *__restrict__ hm, LBDesc<8> *__restrict__ desc,
        unsigned epoch, int write_lists) {
    using word_t = typename Tr<NT>::word_t;
    constexpr int SPT = 128 / NT;
    using BS = cub::BlockScan<Oct, SCAN_BLOCK>;
    __shared__ typename BS::TempStorage ts;
    __shared__ unsigned s_bid;
    __shared__ long long s_pre[8], s_run[4];
    if (threadIdx.x == 0) s_bid = atomicAdd(&cnt->bid_scan, 1u);
    __syncthreads();
    const unsigned bid = s_bid;
    const long long nst = (nseg + (long long)SCAN_BLOCK * SPT - 1) / ((long long)SCAN_BLOCK * SPT);
    const long long t0 = (long long)bid * tpb, t1 = min(nst, t0 + tpb);
    Oct acc;
#pragma unroll
    for (int i = 0; i < 8; ++i) acc.v[i] = 0;
    for (long long t = t0; t < t1; ++t) {
        const long long u = t * SCAN_BLOCK + threadIdx.x;  // this thread's 16-byte unit
        const uint4 f4 = ld_f4<NT>(F, u * 4, nwpad);
        if (f4.x | f4.y | f4.z | f4.w) {
#pragma unroll 1
            for (int k = 0; k < SPT; ++k) {
                const long long J = u * SPT + k;
                if (J >= nseg) break;
                Oct q;
                long long wt;
                scan_seg<NT>(F, J, tptr, sptr, outdeg, indeg, row_begin, m_local, true, q, wt);
#pragma unroll
                for (int i = 0; i < 8; ++i) acc.v[i] += q.v[i];
            }
        }
        // clear the consumed frontier (the level that was just expanded)
        if (Fclear && u * 4 + 4 <= nwpad) *reinterpret_cast<uint4 *>(Fclear + u * 4) = make_uint4(0u, 0u, 0u, 0u);
    }
    if (!write_lists) {
        // statistics only: block reduction + one atomic per value and block; the
        // last block publishes (no look-back chain across blocks)
        __shared__ long long s_red[7];
        __shared__ bool s_last;
        if (threadIdx.x < 7) s_red[threadIdx.x] = 0;
        __syncthreads();
#pragma unroll
        for (int i = 0; i < 7; ++i) {
            long long x = acc.v[i];
#pragma unroll
            for (int o = 16; o > 0; o >>= 1) x += __shfl_xor_sync(0xffffffffu, x, o);
            if ((threadIdx.x & 31) == 0 && x) atomicAdd((unsigned long long *)&s_red[i], (unsigned long long)x);
        }
        __syncthreads();
        if (threadIdx.x == 0) {
            long long *dst[7] = {&cnt->nLt, &cnt->Wt, &cnt->nLs, &cnt->Ws, &cnt->fsize, &cnt->mf, &cnt->din};
            for (int i = 0; i < 7; ++i)
                if (s_red[i]) atomicAdd((unsigned long long *)dst[i], (unsigned long long)s_red[i]);
            __threadfence();
            s_last = atomicAdd(&cnt->fscan_ticket, 1u) == gridDim.x - 1;
        }
        __syncthreads();
        if (s_last && threadIdx.x == 0) {
            __threadfence();
            const long long nLt = __ldcg(&cnt->nLt), Wt = __ldcg(&cnt->Wt), nLs = __ldcg(&cnt->nLs),
                            Ws = __ldcg(&cnt->Ws), fs = __ldcg(&cnt->fsize), mf = __ldcg(&cnt->mf),
                            din = __ldcg(&cnt->din);
            cnt->nCt = (Wt + CHUNK - 1) >> CHUNK_LOG;
            cnt->nCs = (Ws + CHUNK - 1) >> CHUNK_LOG;
            hm->fsize = fs;
            hm->mf = mf;
            hm->din = din;
            hm->nLt = nLt;
            hm->Wt = Wt;
            hm->nLs = nLs;
            hm->Ws = Ws;
            cnt->chunk_next = 0;
            cnt->bid_scan = 0;
            cnt->fscan_ticket = 0;
        }
        return;
    }
    Oct zero, ex, agg;
#pragma unroll
    for (int i = 0; i < 8; ++i) zero.v[i] = 0;
    BS(ts).ExclusiveScan(acc, ex, zero, OctSum(), agg);
    if (threadIdx.x < 32) {
        long long pre[8];
        lookback_warp<8>(desc, bid, epoch, agg.v, pre, threadIdx.x);
        if (threadIdx.x == 0) {
#pragma unroll
            for (int i = 0; i < 8; ++i) s_pre[i] = pre[i];
#pragma unroll
            for (int i = 0; i < 4; ++i) s_run[i] = pre[i];
        }
    }
    __syncthreads();
    for (long long t = t0; t < t1; ++t) {
        const long long u = t * SCAN_BLOCK + threadIdx.x;
        const uint4 f4 = ld_f4<NT>(F, u * 4, nwpad);
        const bool any = (f4.x | f4.y | f4.z | f4.w) != 0u;
        if (!__syncthreads_or(any)) continue;  // no frontier bit in this super-tile
        Oct q;
#pragma unroll
        for (int i = 0; i < 8; ++i) q.v[i] = 0;
        if (any) {
#pragma unroll 1
            for (int k = 0; k < SPT; ++k) {
                const long long J = u * SPT + k;
                if (J >= nseg) break;
                Oct qk;
                long long wt;
                scan_seg<NT>(F, J, tptr, sptr, outdeg, indeg, row_begin, m_local, false, qk, wt);
#pragma unroll
                for (int i = 0; i < 4; ++i) q.v[i] += qk.v[i];
            }
        }
        Oct tagg;
        BS(ts).ExclusiveScan(q, ex, zero, OctSum(), tagg);
        if (any) {
            long long it = s_run[0] + ex.v[0], wp = s_run[1] + ex.v[1];
            long long is = s_run[2] + ex.v[2], w0 = s_run[3] + ex.v[3];
#pragma unroll 1
            for (int k = 0; k < SPT; ++k) {
                const long long J = u * SPT + k;
                if (J >= nseg) break;
                const word_t bits = seg_bits<NT>(F, J);
                if (!bits) continue;
                const long long wt = tptr[J + 1] - tptr[J];
                if (wt > 0) {
                    Lv.Lt_seg[it] = J;
                    Lv.Lt_mask[it] = (unsigned long long)bits;
                    Lv.Lt_tbeg[it] = tptr[J];
                    Lv.Lt_wpre[it] = wp;
                    write_chunks(Lv.Ct, wp, wt, (int)it);
                    ++it;
                    wp += wt;
                }
                word_t b = bits;
                while (b) {
                    int r = ffs_w(b);
                    b &= b - 1;
                    long long v = J * NT + r;
                    long long ws = sptr[v + 1] - sptr[v];
                    if (ws > 0) {
                        Lv.Ls_beg[is] = sptr[v];
                        Lv.Ls_wpre[is] = w0;
                        Lv.Ls_col[is] = (int)v;
                        write_chunks(Lv.Cs, w0, ws, (int)is);
                        ++is;
                        w0 += ws;
                    }
                }
            }
        }
        __syncthreads();  // every thread has read s_run
        if (threadIdx.x < 4) s_run[threadIdx.x] += tagg.v[threadIdx.x];
        __syncthreads();
    }
    if (bid == gridDim.x - 1 && threadIdx.x == 0) {
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

// Statistics-only frontier scan for nt = 16 (hybrid driver after a host pull
// level): thread per HALF segment (8 vertices: 2 + 2 + 4.5 vector loads), grid-
// stride, block reduction + one atomic per value and block, the last block
// publishes; half the registers of k_fscan's whole-segment path, so twice the
// resident threads and no waves.
// LITE (the hybrid driver after a host pull level): only |F|, m_f and the sum of
// in-degrees, which its direction decision reads (the work totals are recounted
// by the persistent kernel when it resumes); a symmetric pattern's in-degrees are
// its out-degrees (one array read).
// The lite statistics of a symmetric single-GPU context (in-degrees == out-degrees):
// thread per 32-vertex word of F, two words per step, each non-zero word's 32
// degrees as eight 16-byte loads (one line, all in flight); clears Fclear.
__global__ void __launch_bounds__(256) k_fstats_words(const uint32_t *__restrict__ F, uint32_t *__restrict__ Fclear,
                                                      long long nw, const int *__restrict__ deg,
                                                      Counters *__restrict__ cnt, Counters *__restrict__ hm) {
    const long long S = (long long)gridDim.x * blockDim.x;
    unsigned long long f = 0, mf = 0;
    for (long long w0 = blockIdx.x * (long long)blockDim.x + threadIdx.x; w0 < nw; w0 += 2 * S) {
        uint32_t b[2];
#pragma unroll
        for (int k = 0; k < 2; ++k) {
            const long long w = w0 + k * S;
            b[k] = w < nw ? __ldcg(&F[w]) : 0u;
            if (Fclear && w < nw) Fclear[w] = 0u;
        }
#pragma unroll
        for (int k = 0; k < 2; ++k) {
            if (!b[k]) continue;
            const int4 *dp = reinterpret_cast<const int4 *>(deg + (w0 + k * S) * 32);
            int4 d[8];
#pragma unroll
            for (int i = 0; i < 8; ++i) d[i] = __ldg(dp + i);
            f += (unsigned long long)__popc(b[k]);
#pragma unroll
            for (int i = 0; i < 8; ++i) {
                const unsigned m4 = b[k] >> (4 * i);
                if (m4 & 1u) mf += (unsigned long long)d[i].x;
                if (m4 & 2u) mf += (unsigned long long)d[i].y;
                if (m4 & 4u) mf += (unsigned long long)d[i].z;
                if (m4 & 8u) mf += (unsigned long long)d[i].w;
            }
        }
    }
    __shared__ unsigned long long s2[2];
    __shared__ bool s_last;
    if (threadIdx.x < 2) s2[threadIdx.x] = 0;
    __syncthreads();
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        f += __shfl_xor_sync(0xffffffffu, f, o);
        mf += __shfl_xor_sync(0xffffffffu, mf, o);
    }
    if ((threadIdx.x & 31) == 0 && f) {
        atomicAdd(&s2[0], f);
        atomicAdd(&s2[1], mf);
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        if (s2[0]) {
            atomicAdd((unsigned long long *)&cnt->fsize, s2[0]);
            atomicAdd((unsigned long long *)&cnt->mf, s2[1]);
        }
        __threadfence();
        s_last = atomicAdd(&cnt->fscan_ticket, 1u) == gridDim.x - 1;
    }
    __syncthreads();
    if (s_last && threadIdx.x == 0) {
        __threadfence();
        const long long fs = __ldcg(&cnt->fsize), m = __ldcg(&cnt->mf);
        hm->fsize = fs;
        hm->mf = m;
        hm->din = m;
        cnt->fscan_ticket = 0;
    }
}

template <bool LITE>
__global__ void __launch_bounds__(256) k_fstats16(const uint32_t *__restrict__ F, uint32_t *__restrict__ Fclear,
                                                  long long nseg, const long long *__restrict__ tptr,
                                                  const long long *__restrict__ sptr, const int *__restrict__ outdeg,
                                                  const int *__restrict__ indeg, long long row_begin,
                                                  long long m_local, Counters *__restrict__ cnt,
                                                  Counters *__restrict__ hm) {
    long long q[7] = {0, 0, 0, 0, 0, 0, 0};
    const long long nh = nseg * 2;
    for (long long hs = blockIdx.x * (long long)blockDim.x + threadIdx.x; hs < nh;
         hs += (long long)gridDim.x * blockDim.x) {
        const long long J = hs >> 1;
        const int h = (int)(hs & 1);
        const uint32_t w = F[J >> 1];
        const unsigned bits8 = (w >> (((J & 1) << 4) + (h << 3))) & 0xffu;
        if (h == 0 && Fclear && (J & 1) == 0) Fclear[J >> 1] = 0u;
        if (!bits8) continue;
        if (!LITE && (h == 0 || !((w >> ((J & 1) << 4)) & 0xffu))) {
            // tile work of the segment, counted once: by the low half, or by the
            // high half when the low half is empty
            const long long wt = tptr[J + 1] - tptr[J];
            q[0] += wt > 0;
            q[1] += wt;
        }
        const long long v0 = J * 16 + h * 8;
        int od[8], id[8];
        long long sp[9];
        const int4 o0 = __ldg(reinterpret_cast<const int4 *>(outdeg + v0)),
                   o1 = __ldg(reinterpret_cast<const int4 *>(outdeg + v0) + 1);
        od[0] = o0.x, od[1] = o0.y, od[2] = o0.z, od[3] = o0.w, od[4] = o1.x, od[5] = o1.y, od[6] = o1.z, od[7] = o1.w;
        if (!LITE) {
#pragma unroll
            for (int i = 0; i < 4; ++i) {
                const longlong2 t = __ldg(reinterpret_cast<const longlong2 *>(sptr + v0) + i);
                sp[2 * i] = t.x, sp[2 * i + 1] = t.y;
            }
            sp[8] = __ldg(sptr + v0 + 8);
        } else {
#pragma unroll
            for (int i = 0; i < 9; ++i) sp[i] = 0;
        }
        const long long lv0 = v0 - row_begin;
        if (LITE && indeg == outdeg && row_begin == 0) {
#pragma unroll
            for (int r = 0; r < 8; ++r) id[r] = od[r];
        } else if (lv0 >= 0 && lv0 + 8 <= m_local) {
            const int4 i0 = __ldg(reinterpret_cast<const int4 *>(indeg + lv0)),
                       i1 = __ldg(reinterpret_cast<const int4 *>(indeg + lv0) + 1);
            id[0] = i0.x, id[1] = i0.y, id[2] = i0.z, id[3] = i0.w, id[4] = i1.x, id[5] = i1.y, id[6] = i1.z,
            id[7] = i1.w;
        } else {
#pragma unroll
            for (int r = 0; r < 8; ++r) id[r] = (lv0 + r >= 0 && lv0 + r < m_local) ? __ldg(indeg + lv0 + r) : 0;
        }
        q[4] += __popc(bits8);
#pragma unroll
        for (int r = 0; r < 8; ++r) {
            if ((bits8 >> r) & 1u) {
                const long long ws = sp[r + 1] - sp[r];
                q[2] += ws > 0;
                q[3] += ws;
                q[5] += od[r];
                q[6] += id[r];
            }
        }
    }
    __shared__ unsigned long long s_red[7];
    __shared__ bool s_last;
    if (threadIdx.x < 7) s_red[threadIdx.x] = 0;
    __syncthreads();
#pragma unroll
    for (int i = 0; i < 7; ++i) {
        long long x = q[i];
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) x += __shfl_xor_sync(0xffffffffu, x, o);
        if ((threadIdx.x & 31) == 0 && x) atomicAdd(&s_red[i], (unsigned long long)x);
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        long long *dst[7] = {&cnt->nLt, &cnt->Wt, &cnt->nLs, &cnt->Ws, &cnt->fsize, &cnt->mf, &cnt->din};
        for (int i = 0; i < 7; ++i)
            if (s_red[i]) atomicAdd((unsigned long long *)dst[i], s_red[i]);
        __threadfence();
        s_last = atomicAdd(&cnt->fscan_ticket, 1u) == gridDim.x - 1;
    }
    __syncthreads();
    if (s_last && threadIdx.x == 0) {
        __threadfence();
        hm->fsize = __ldcg(&cnt->fsize);
        hm->mf = __ldcg(&cnt->mf);
        hm->din = __ldcg(&cnt->din);
        hm->nLt = __ldcg(&cnt->nLt);
        hm->Wt = __ldcg(&cnt->Wt);
        hm->nLs = __ldcg(&cnt->nLs);
        hm->Ws = __ldcg(&cnt->Ws);
        cnt->chunk_next = 0;
        cnt->fscan_ticket = 0;
    }
}

// Push (vector-driven): tile chunks (Push-CSC, Alg 5) and side chunks.
template <int NT, bool DO_TILES>
__global__ void __launch_bounds__(256)
k_push(BfsTiles P, ListsView Lv, Counters *__restrict__ cnt, BfsView B, int bulk_ok) {
    __shared__ long long win_all[8][CHUNK + 1];
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    long long *win = win_all[wid];
    const long long nCt = DO_TILES ? cnt->nCt : 0, nCs = cnt->nCs;
    const long long nLt = cnt->nLt, nLs = cnt->nLs, Wt = cnt->Wt, Ws = cnt->Ws;
    const bool bulk = bulk_ok && push_bulk(DO_TILES, Wt, Ws, B.m_local);  // k_bulk_fix finishes the level
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
                push_tile_item<NT>(P, B, Lv.Lt_tbeg[s] + (i - win[q]), (typename Tr<NT>::word_t)Lv.Lt_mask[s],
                                   bulk);
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
                push_side_item<NT>(P, B, Lv.Ls_beg[s0 + q] + (i - win[q]), bulk);
            }
            __syncwarp();
        } else {
            break;
        }
    }
}

// Bulk Push-CSC level (r2, as the fused kernel's): k_push only ORed the reached
// rows into Fn; over this rank's words new = Fn & ~V, V |= new, levels (a no-op
// when the level was not bulk: same test on the same counters)
__global__ void k_bulk_fix(const Counters *__restrict__ cnt, BfsView B) {
    if (!push_bulk(true, cnt->Wt, cnt->Ws, B.m_local)) return;
    const long long w0 = B.row_begin >> 5, w1 = (B.row_begin + B.m_local + 31) >> 5;
    for (long long w = w0 + blockIdx.x * (long long)blockDim.x + threadIdx.x; w < w1;
         w += (long long)gridDim.x * blockDim.x) {
        const uint32_t f = B.Fn[w];
        if (!f) continue;
        const uint32_t v = B.V[w];
        const uint32_t nw = f & ~v;
        B.Fn[w] = nw;
        if (nw) {
            B.V[w] = v | nw;
            uint32_t bb = nw;
            while (bb) {
                const int r = __ffs(bb) - 1;
                bb &= bb - 1;
                B.levels[w * 32 + r - B.row_begin] = B.level + 1;
            }
        }
    }
}

template <int NT>
__global__ void __launch_bounds__(256) k_push_csr(BfsTiles Q, BfsView B) {
    for (long long t = blockIdx.x * (long long)blockDim.x + threadIdx.x; t < Q.T;
         t += (long long)gridDim.x * blockDim.x)
        push_csr_item<NT>(Q, B, t);
}

// WIDE (late pull levels, few open rows): a warp tests the visited words of 32
// row tiles at once and walks only the open ones; otherwise warp per row tile.
// Dense Pull-CSC level, tile part, W lanes per row tile (32 / W row tiles per
// warp walked together: the warp's rounds run while any of its row tiles still
// has tiles and unvisited rows; W = 32 is k_pull's one row tile per warp).
template <int NT, int W>
__global__ void __launch_bounds__(256) k_pull_sub(BfsTiles Q, BfsView B, long long nTR_local) {
    using word_t = typename Tr<NT>::word_t;
    constexpr int R = 32 / W;
    const word_t *planes = (const word_t *)Q.planes;
    const int lane = threadIdx.x & 31, gl = lane % W, grp = lane / W;
    const long long warp = (blockIdx.x * (long long)blockDim.x + threadIdx.x) >> 5;
    const long long nwarps = ((long long)gridDim.x * blockDim.x) >> 5;
    const long long rb_seg = B.row_begin / NT;
    for (long long I0 = warp * R; I0 < nTR_local; I0 += nwarps * R) {
        const long long I = I0 + grp;
        word_t um = 0;
        long long tb = 0, t1 = 0;
        if (I < nTR_local) {
            um = ~seg_bits<NT>(B.V, rb_seg + I) & (word_t)Q.pmask[I];
            if (um) {
                tb = Q.ptr[I];
                t1 = Q.ptr[I + 1];
            }
        }
        word_t found = 0;
        while (__any_sync(0xffffffffu, um && tb < t1)) {
            const long long t = tb + gl;
            word_t fl = 0;
            if (um && t < t1) {
                const word_t f = seg_bits<NT>(B.F, Q.trow[t]);
                if (f) fl = rows_hit<NT>(planes, Q.T, t, um, f);
            }
#pragma unroll
            for (int o = W / 2; o > 0; o >>= 1) fl |= (word_t)__shfl_xor_sync(0xffffffffu, fl, o);
            found |= fl;
            um &= ~fl;
            tb += W;
        }
        if (gl == 0 && found) discover<NT>(B, rb_seg + I, found);
    }
}

template <int NT, bool WIDE>
__global__ void __launch_bounds__(256) k_pull(BfsTiles Q, BfsView B, long long nTR_local) {
    const int lane = threadIdx.x & 31;
    const long long warp = (blockIdx.x * (long long)blockDim.x + threadIdx.x) >> 5;
    const long long nwarps = ((long long)gridDim.x * blockDim.x) >> 5;
    if constexpr (WIDE) {
        for (long long I0 = warp * 32; I0 < nTR_local; I0 += nwarps * 32) pull_rowtiles32<NT>(Q, B, I0, nTR_local, lane);
    } else {
        for (long long I = warp; I < nTR_local; I += nwarps) pull_rowtile<NT>(Q, B, I, lane);
    }
}

template <int NT, bool WIDE>
__global__ void __launch_bounds__(256) k_pull_side(BfsTiles Q, BfsView B) {
    if constexpr (WIDE) {  // thread per visited word: one load for 32 settled vertices
        const long long w0 = B.row_begin / 32, nw = (B.m_local + 31) / 32;
        for (long long w = blockIdx.x * (long long)blockDim.x + threadIdx.x; w < nw;
             w += (long long)gridDim.x * blockDim.x)
            pull_side_word<NT>(Q, B, w0 + w);
    } else {
        for (long long v = blockIdx.x * (long long)blockDim.x + threadIdx.x; v < B.m_local;
             v += (long long)gridDim.x * blockDim.x)
            pull_side_vertex<NT>(Q, B, v);
    }
}

// Dense Pull-CSC level, side part, K vertices per thread (v0, v0 + S, ..., S =
// the grid's threads): every dependent step (visited + side-mask words, the
// row's range, PR in-neighbour ids, their frontier bits, the claim on V) is
// issued for all K vertices before the next, so K chains of loads are in flight
// per thread instead of one; vertices whose row ends or hits drop out of the
// rounds.  Same result as k_pull_side<NT, false> (every vertex of the level is
// tested against the frontier snapshot F, claimed with an atomic on V).
template <int NT, int K>
__global__ void __launch_bounds__(256) k_pull_side_ilp(BfsTiles Q, BfsView B) {
#ifndef TSMV_PULL_ROUND
#define TSMV_PULL_ROUND 2
#endif
    constexpr int PR = TSMV_PULL_ROUND;
    const int lane = threadIdx.x & 31;
    const long long S = (long long)gridDim.x * blockDim.x;
    // warp-uniform loop: lane l takes vertex wb + l (+ k S), so the warp's vertices
    // of step k are one aligned 32-bit word of V (row_begin is a multiple of 64)
    for (long long wb = blockIdx.x * (long long)blockDim.x + (threadIdx.x & ~31); wb < B.m_local; wb += S * K) {
        const long long v0 = wb + lane;
        uint32_t vw[K], sw[K];
#pragma unroll
        for (int k = 0; k < K; ++k) {
            const long long v = v0 + k * S;
            vw[k] = 0xffffffffu;
            sw[k] = 0u;
            if (v < B.m_local) {
                vw[k] = B.V[(B.row_begin + v) >> 5];
                sw[k] = Q.smask[v >> 5];
            }
        }
        unsigned act = 0u;
#pragma unroll
        for (int k = 0; k < K; ++k) {
            const long long v = v0 + k * S, g = B.row_begin + v;
            if (v < B.m_local && !((vw[k] >> (g & 31)) & 1u) && ((sw[k] >> (v & 31)) & 1u)) act |= 1u << k;
        }
        long long p[K], pe[K];
#pragma unroll
        for (int k = 0; k < K; ++k) {
            p[k] = pe[k] = 0;
            if ((act >> k) & 1u) {
                p[k] = Q.sptr[v0 + k * S];
                pe[k] = Q.sptr[v0 + k * S + 1];
            }
        }
        unsigned found = 0u;
        while (act) {
            int sr[K][PR];
#pragma unroll
            for (int k = 0; k < K; ++k)
#pragma unroll
                for (int j = 0; j < PR; ++j) sr[k][j] = ((act >> k) & 1u) && p[k] + j < pe[k] ? Q.srow[p[k] + j] : 0;
            bool hit[K];
#pragma unroll
            for (int k = 0; k < K; ++k) {
                hit[k] = false;
                if ((act >> k) & 1u)
#pragma unroll
                    for (int j = 0; j < PR; ++j)
                        if (p[k] + j < pe[k]) {
                            const long long u = decode_row<NT>(sr[k][j], Q.hot_list);
                            hit[k] |= ((B.F[u >> 5] >> (u & 31)) & 1u) != 0;
                        }
            }
#pragma unroll
            for (int k = 0; k < K; ++k) {
                if (!((act >> k) & 1u)) continue;
                if (hit[k]) {
                    found |= 1u << k;
                    act &= ~(1u << k);
                } else {
                    p[k] += PR;
                    if (p[k] >= pe[k]) act &= ~(1u << k);
                }
            }
        }
        // claims: one atomic per (warp, word) with the warp's ballot (dense pull
        // levels discover most vertices: 32x fewer same-word atomics on V), all K
        // in flight; then the new vertices' frontier bits (one reduction per word)
        // and levels
        unsigned bal[K], old[K];
#pragma unroll
        for (int k = 0; k < K; ++k) bal[k] = __ballot_sync(0xffffffffu, (found >> k) & 1u);
#pragma unroll
        for (int k = 0; k < K; ++k) {
            old[k] = 0u;
            if (lane == 0 && bal[k]) old[k] = atomicOr(&B.V[(B.row_begin + wb + k * S) >> 5], bal[k]);
        }
#pragma unroll
        for (int k = 0; k < K; ++k) {
            if (!bal[k]) continue;
            const unsigned nw = bal[k] & ~__shfl_sync(0xffffffffu, old[k], 0);
            if (lane == 0 && nw) atomicOr(&B.Fn[(B.row_begin + wb + k * S) >> 5], nw);
            if ((nw >> lane) & 1u) B.levels[v0 + k * S] = B.level + 1;
        }
    }
}

// BFS parents over the min-second semiring:
// parent[v] = min { u : edge u -> v (A[v][u] stored), levels[u] = levels[v] - 1 },
// parent[source] = source, -1 if unreachable.  One warp per vertex: the lanes
// walk v's row words in the row structure Q (tiles ascending by tile column, so
// the first round of 32 tiles with a candidate holds the smallest one), then
// v's side row, keeping the minimum.
template <int NT>
__global__ void __launch_bounds__(256) k_parents(BfsTiles Q, const int32_t *__restrict__ levels,
                                                 int32_t *__restrict__ parents, long long m) {
    using word_t = typename Tr<NT>::word_t;
    const word_t *planes = (const word_t *)Q.planes;
    const int lane = threadIdx.x & 31;
    const long long warp = (blockIdx.x * (long long)blockDim.x + threadIdx.x) >> 5;
    const long long nwarps = ((long long)gridDim.x * blockDim.x) >> 5;
    for (long long v = warp; v < m; v += nwarps) {
        const int L = levels[v];
        if (L <= 0) {
            if (lane == 0) parents[v] = (L == 0) ? (int32_t)v : -1;
            continue;
        }
        const long long I = v / NT;
        const int r = (int)(v % NT);
        int best = INT_MAX;
        const long long t0 = Q.ptr[I], t1 = Q.ptr[I + 1];
        for (long long tb = t0; tb < t1 && best == INT_MAX; tb += 32) {
            const long long t = tb + lane;
            int cand = INT_MAX;
            if (t < t1) {
                word_t w = planes[(long long)r * Q.T + t];
                const long long base = (long long)Q.trow[t] * NT;
                while (w) {
                    const int c = ffs_w(w);
                    w &= w - 1;
                    if (levels[base + c] == L - 1) {
                        cand = (int)(base + c);
                        break;
                    }
                }
            }
            best = __reduce_min_sync(0xffffffffu, cand);
        }
        int sb = best;
        for (long long p = Q.sptr[v] + lane; p < Q.sptr[v + 1]; p += 32) {
            const long long u = decode_row<NT>(Q.srow[p], Q.hot_list);
            if (u < sb && levels[u] == L - 1) sb = (int)u;
        }
        sb = __reduce_min_sync(0xffffffffu, sb);
        if (lane == 0) parents[v] = sb == INT_MAX ? -1 : sb;
    }
}

// nt = 16 parents in two passes.  Tile part: warp per row tile I (16 rows at
// once); lanes walk the tiles of the group in ascending tile-column order, every
// lane loads the 16 row words of its tile (predicated, one round) and keeps,
// per row, the first in-neighbour c (ascending) at the previous level; a warp
// min per row over the first round of 32 tiles with any candidate gives the
// row's smallest tile-part parent.  Side part: thread per vertex (warp per
// vertex above 64 side in-neighbours), minimum over the side row.
__global__ void __launch_bounds__(256) k_parents_tiles16(BfsTiles Q, const int32_t *__restrict__ levels,
                                                         int32_t *__restrict__ parents, long long m, long long nTR) {
    const uint16_t *planes = (const uint16_t *)Q.planes;
    const int lane = threadIdx.x & 31;
    const long long warp = (blockIdx.x * (long long)blockDim.x + threadIdx.x) >> 5;
    const long long nwarps = ((long long)gridDim.x * blockDim.x) >> 5;
    for (long long I = warp; I < nTR; I += nwarps) {
        const long long v0 = I * 16;
        const int L = (lane < 16 && v0 + lane < m) ? levels[v0 + lane] : -1;
        // rows that need a parent: level > 0 (lane r holds row r's level)
        unsigned need = __ballot_sync(0xffffffffu, L > 0) & 0xffffu;
        int lvl[16];
#pragma unroll
        for (int r = 0; r < 16; ++r) lvl[r] = __shfl_sync(0xffffffffu, L, r);
        int best[16];
#pragma unroll
        for (int r = 0; r < 16; ++r) best[r] = INT_MAX;
        const long long t0 = Q.ptr[I], t1 = Q.ptr[I + 1];
        for (long long tb = t0; tb < t1 && need; tb += 32) {
            const long long t = tb + lane;
            int cand[16];
#pragma unroll
            for (int r = 0; r < 16; ++r) cand[r] = INT_MAX;
            if (t < t1) {
                const long long base = (long long)Q.trow[t] * 16;
                unsigned w[16];
#pragma unroll
                for (int r = 0; r < 16; ++r) w[r] = ((need >> r) & 1u) ? planes[(long long)r * Q.T + t] : 0u;
#pragma unroll
                for (int r = 0; r < 16; ++r) {
                    unsigned x = w[r];
                    while (x) {
                        const int c = __ffs(x) - 1;
                        x &= x - 1;
                        if (levels[base + c] == lvl[r] - 1) {
                            cand[r] = (int)(base + c);
                            break;
                        }
                    }
                }
            }
            unsigned found = 0;
#pragma unroll
            for (int r = 0; r < 16; ++r) {
                if ((need >> r) & 1u) {  // uniform
                    const int mn = __reduce_min_sync(0xffffffffu, cand[r]);
                    if (mn != INT_MAX) {
                        best[r] = mn;
                        found |= 1u << r;
                    }
                }
            }
            need &= ~found;  // rows with a tile-part parent in this round are done
        }
        if (lane < 16 && v0 + lane < m) {
            int bl = INT_MAX;
#pragma unroll
            for (int r = 0; r < 16; ++r)
                if (r == lane) bl = best[r];
            parents[v0 + lane] = L == 0 ? (int32_t)(v0 + lane) : (L < 0 ? -1 : bl);
        }
    }
}

template <int NT, bool WARP>
__global__ void __launch_bounds__(256) k_parents_side(BfsTiles Q, const int32_t *__restrict__ levels,
                                                      int32_t *__restrict__ parents, long long m) {
    const int lane = threadIdx.x & 31;
    const long long tid = blockIdx.x * (long long)blockDim.x + threadIdx.x;
    const long long nt = (long long)gridDim.x * blockDim.x;
    const long long first = WARP ? (tid >> 5) : tid, stride = WARP ? (nt >> 5) : nt;
    for (long long v = first; v < m; v += stride) {
        if (!((Q.smask[v >> 5] >> (v & 31)) & 1u)) continue;
        const long long p0 = Q.sptr[v], p1 = Q.sptr[v + 1];
        if ((p1 - p0 > 32) != WARP) continue;
        const int L = levels[v];
        if (L <= 0) continue;
        int cur = parents[v];
        int sb = cur;
        if (WARP) {
            for (long long p = p0 + lane; p < p1; p += 32) {
                const long long u = decode_row<NT>(Q.srow[p], Q.hot_list);
                if (u < sb && levels[u] == L - 1) sb = (int)u;
            }
            sb = __reduce_min_sync(0xffffffffu, sb);
            if (lane == 0 && sb < cur) parents[v] = sb;
        } else {
            for (long long p = p0; p < p1; p += 4) {  // 4 in-neighbours, then their levels, per round
                long long u[4];
#pragma unroll
                for (int j = 0; j < 4; ++j) u[j] = p + j < p1 ? decode_row<NT>(Q.srow[p + j], Q.hot_list) : -1;
                int lv[4];
#pragma unroll
                for (int j = 0; j < 4; ++j) lv[j] = (u[j] >= 0 && u[j] < sb) ? levels[u[j]] : -2;
#pragma unroll
                for (int j = 0; j < 4; ++j)
                    if (lv[j] == L - 1 && u[j] < sb) sb = (int)u[j];
            }
            if (sb < cur) parents[v] = sb;
        }
    }
}

// heavy side rows (> 64 in-neighbours, power-law hubs) in chunks of 256
// entries, one warp per chunk, combined with atomicMin
constexpr int PAR_CHUNK = 256;
__global__ void k_par_chunk_count(const long long *__restrict__ sptr, long long m, int *__restrict__ cnt) {
    for (long long v = blockIdx.x * (long long)blockDim.x + threadIdx.x; v < m; v += (long long)gridDim.x * blockDim.x) {
        const long long len = sptr[v + 1] - sptr[v];
        cnt[v] = len > 32 ? (int)((len + PAR_CHUNK - 1) / PAR_CHUNK) : 0;
    }
}
__global__ void k_par_chunk_fill(const long long *__restrict__ sptr, long long m, const long long *__restrict__ off,
                                 const int *__restrict__ cnt, long long *__restrict__ chunks) {
    for (long long v = blockIdx.x * (long long)blockDim.x + threadIdx.x; v < m; v += (long long)gridDim.x * blockDim.x)
        for (int i = 0; i < cnt[v]; ++i) chunks[off[v] + i] = (v << 24) | (long long)i;  // v < 2^39, chunk < 2^24
}
template <int NT>
__global__ void __launch_bounds__(256) k_parents_chunks(BfsTiles Q, const int32_t *__restrict__ levels,
                                                        int32_t *__restrict__ parents, const long long *__restrict__ chunks,
                                                        long long nchunks) {
    const int lane = threadIdx.x & 31;
    const long long warp = (blockIdx.x * (long long)blockDim.x + threadIdx.x) >> 5;
    const long long nwarps = ((long long)gridDim.x * blockDim.x) >> 5;
    for (long long q = warp; q < nchunks; q += nwarps) {
        const long long e = chunks[q];
        const long long v = e >> 24, i = e & 0xffffff;
        const int L = levels[v];
        if (L <= 0) continue;
        const long long p0 = Q.sptr[v] + i * PAR_CHUNK, p1 = min(Q.sptr[v + 1], p0 + PAR_CHUNK);
        int sb = INT_MAX;
        for (long long p = p0 + lane; p < p1; p += 32) {
            const long long u = decode_row<NT>(Q.srow[p], Q.hot_list);
            if (u < sb && levels[u] == L - 1) sb = (int)u;
        }
        sb = __reduce_min_sync(0xffffffffu, sb);
        if (lane == 0 && sb != INT_MAX) atomicMin(&parents[v], sb);
    }
}

__global__ void k_parents_fix(int32_t *__restrict__ parents, long long m) {
    for (long long v = blockIdx.x * (long long)blockDim.x + threadIdx.x; v < m; v += (long long)gridDim.x * blockDim.x)
        if (parents[v] == INT_MAX) parents[v] = -1;
}


// Statistics of this rank's share of the next frontier (distributed levels, r2):
// over the owned words [w0, w1) of F: out[0] += |F_owned|, out[1] += sum of the
// GLOBAL out-degrees of those vertices (m_f share), out[2] += sum of their
// in-degrees (row counts of owned rows: the m_u decrement).  Every rank scans
// only its own rows, O(n / P); the shares are summed over the ranks.
__global__ void k_owned_stats(const uint32_t *__restrict__ F, long long w0, long long w1, long long row_begin,
                              const int *__restrict__ outdeg_g, const int *__restrict__ indeg_local,
                              unsigned long long *__restrict__ out) {
    // a warp takes 32 consecutive words (one coalesced load), then walks them:
    // for a non-zero word lane l tests bit l, so the degree loads of a word are
    // one 128-byte line each (a thread-per-word bit loop serialised them)
    const int lane = threadIdx.x & 31;
    const long long nwarps = ((long long)gridDim.x * blockDim.x) >> 5;
    unsigned long long q0 = 0, q1 = 0, q2 = 0;
    for (long long wb = w0 + (((long long)blockIdx.x * blockDim.x + threadIdx.x) >> 5) * 32; wb < w1;
         wb += nwarps * 32) {
        const uint32_t mine = (wb + lane < w1) ? __ldg(F + wb + lane) : 0u;
        unsigned nz = __ballot_sync(0xffffffffu, mine != 0u);
        while (nz) {
            const int j = __ffs(nz) - 1;
            nz &= nz - 1;
            const uint32_t b = __shfl_sync(0xffffffffu, mine, j);
            if ((b >> lane) & 1u) {
                const long long v = (wb + j) * 32 + lane;
                ++q0;
                q1 += (unsigned long long)__ldg(outdeg_g + v);
                q2 += (unsigned long long)__ldg(indeg_local + (v - row_begin));
            }
        }
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        q0 += __shfl_xor_sync(0xffffffffu, q0, o);
        q1 += __shfl_xor_sync(0xffffffffu, q1, o);
        q2 += __shfl_xor_sync(0xffffffffu, q2, o);
    }
    if (lane == 0 && q0) {
        atomicAdd(&out[0], q0);
        atomicAdd(&out[1], q1);
        atomicAdd(&out[2], q2);
    }
}
// begin: shares of the source's frontier {source} (only its owner counts it)
__global__ void k_source_stats(long long source, long long row_begin, long long m_local,
                               const int *__restrict__ outdeg_g, const int *__restrict__ indeg_local,
                               unsigned long long *__restrict__ out) {
    const bool own = source >= row_begin && source < row_begin + m_local;
    out[0] = own ? 1ull : 0ull;
    out[1] = own ? (unsigned long long)outdeg_g[source] : 0ull;
    out[2] = own ? (unsigned long long)indeg_local[source - row_begin] : 0ull;
}
// distributed merge with device statistics: {|F| share, m_f share, m_u local}
__global__ void k_dist_stats2(const unsigned long long *__restrict__ dstats, long long *__restrict__ mu,
                              int64_t *__restrict__ out) {
    const long long m = *mu - (long long)dstats[2];
    *mu = m;
    out[0] = (long long)dstats[0];
    out[1] = (long long)dstats[1];
    out[2] = m;
}

// 2D block level prologue (tsmv_bfs2d_expand)
__global__ void k_level2d_prep(uint32_t *__restrict__ V, const uint32_t *__restrict__ rnew, uint32_t *__restrict__ Fn,
                               long long nwr, uint32_t *__restrict__ F, const uint32_t *__restrict__ x, long long nwx,
                               long long nwpad) {
    for (long long w = blockIdx.x * (long long)blockDim.x + threadIdx.x; w < max(nwr, nwpad);
         w += (long long)gridDim.x * blockDim.x) {
        if (w < nwr) {
            if (rnew) {
                const uint32_t b = rnew[w];
                if (b) V[w] |= b;
            }
            Fn[w] = 0u;
        }
        if (w < nwpad) F[w] = w < nwx ? x[w] : 0u;
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
    const BfsView *ov = nullptr;  // 2D block levels: caller-provided row / column bitmaps

    BfsView view() {
        if (ov) return *ov;
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

    // degree arrays of the frontier statistics: a context with its own
    // communicator uses the replicated GLOBAL arrays (every rank then computes
    // the same |F|, m_f and sum of in-degrees from the same frontier bitmap);
    // otherwise its local ones (sum of in-degrees over its own rows only)
    const int *odeg() const { return c->outdeg_g.p ? c->outdeg_g.as<int>() : c->outdeg.as<int>(); }
    const int *ideg() const { return c->indeg_g.p ? c->indeg_g.as<int>() : c->indeg.as<int>(); }
    long long irb() const { return c->indeg_g.p ? 0 : c->row_begin; }
    long long iml() const { return c->indeg_g.p ? c->n : c->m; }

    template <int NT> void fscan(const uint32_t *F, uint32_t *Fclear, bool lists, bool lite = false) {
        long long nseg = c->nTC;
        // one wave: blocks x tiles-per-block cover the ceil(nseg / SCAN_BLOCK) tiles
        static int bps_scan[3] = {0, 0, 0};
        int &bps = bps_scan[NT == 16 ? 0 : NT == 32 ? 1 : 2];
        if (bps == 0 && (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&bps, k_fscan<NT>, SCAN_BLOCK, 0) !=
                             cudaSuccess || bps < 1)) {
            cudaGetLastError();
            bps = 1;
        }
        const long long spt = 128 / NT;
        const long long ntiles = std::max<long long>(1, (nseg + SCAN_BLOCK * spt - 1) / (SCAN_BLOCK * spt));
        const long long cap = std::max<long long>(1, (long long)c->sm_count * bps);
        const long long tpb = (ntiles + cap - 1) / cap;
        const int grid = (int)((ntiles + tpb - 1) / tpb);
        c->epoch++;
        if (!lists)  // the stats-only scan accumulates into zeroed counters {nLt..din}
            TSMV_CUDA(cudaMemsetAsync(&c->counters.as<Counters>()->nLt, 0, 9 * sizeof(long long), st));
        if (!lists && NT == 16) {
            int bps = 0;
            if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&bps, k_fstats16<false>, 256, 0) != cudaSuccess ||
                bps < 1) {
                cudaGetLastError();
                bps = 1;
            }
            const int g = (int)std::max<long long>(
                1, std::min<long long>((nseg * 2 + 255) / 256, (long long)c->sm_count * bps));
            // symmetric pattern: in-degrees == out-degrees (one array)
            const int *id = (c->symmetric && !c->indeg_g.p && !c->outdeg_g.p) ? odeg() : ideg();
            if (lite && c->symmetric && !c->indeg_g.p && !c->outdeg_g.p && c->row_begin == 0 &&
                !getenv("TSMV_BFS_FULL_FSTATS") && !getenv("TSMV_BFS_FSTATS16")) {
                const long long nw = (c->n + 31) / 32;
                k_fstats_words<<<grid_for((nw + 1) / 2), 256, 0, st>>>(F, Fclear, nw, odeg(), c->counters.as<Counters>(),
                                                                      c->hcnt_dev);
            } else if (lite && !getenv("TSMV_BFS_FULL_FSTATS"))
                k_fstats16<true><<<g, 256, 0, st>>>(F, Fclear, nseg, c->P.ptr.as<long long>(),
                                                    c->P.sptr.as<long long>(), odeg(), id, irb(), iml(),
                                                    c->counters.as<Counters>(), c->hcnt_dev);
            else
                k_fstats16<false><<<g, 256, 0, st>>>(F, Fclear, nseg, c->P.ptr.as<long long>(),
                                                     c->P.sptr.as<long long>(), odeg(), ideg(), irb(), iml(),
                                                     c->counters.as<Counters>(), c->hcnt_dev);
            TSMV_CUDA(cudaGetLastError());
            return;
        }
        k_fscan<NT><<<grid, SCAN_BLOCK, 0, st>>>(F, Fclear, nseg, tpb, (long long)(c->V.bytes / 4),
                                                 c->P.ptr.as<long long>(),
                                                 c->P.sptr.as<long long>(), odeg(), ideg(),
                                                 irb(), iml(), lists_view(c), c->counters.as<Counters>(),
                                                 c->hcnt_dev, c->desc_bfs.as<LBDesc<8>>(), c->epoch, lists ? 1 : 0);
        TSMV_CUDA(cudaGetLastError());
    }

    // side part of a dense pull level: K vertices per thread (TSMV_PULL_ILP = 1, 2,
    // 4 or 8; 1 = the thread-per-vertex kernel)
    template <int NT> void pull_side_dense(const BfsTiles &Q, const BfsView &B, cudaStream_t s) {
        // (the warp's word-aligned claims need row_begin % 32 == 0: always true for
        // row blocks, which are cut at multiples of 64)
        const int K = (B.row_begin & 31) ? 0 : getenv("TSMV_PULL_ILP") ? atoi(getenv("TSMV_PULL_ILP")) : 1;
        const long long m = c->m;
        if (K == 8) k_pull_side_ilp<NT, 8><<<grid_for((m + 7) / 8), 256, 0, s>>>(Q, B);
        else if (K == 4) k_pull_side_ilp<NT, 4><<<grid_for((m + 3) / 4), 256, 0, s>>>(Q, B);
        else if (K == 2) k_pull_side_ilp<NT, 2><<<grid_for((m + 1) / 2), 256, 0, s>>>(Q, B);
        else if (K == 1) k_pull_side_ilp<NT, 1><<<grid_for(m), 256, 0, s>>>(Q, B);
        else k_pull_side<NT, false><<<grid_for(m), 256, 0, s>>>(Q, B);
    }

    // tile part of a dense pull level: W lanes per row tile, 32 / W row tiles per
    // warp (TSMV_PULL_W = 4 | 8 | 16 | 32; 32 = k_pull, r2).  Measured (session 5,
    // R-MAT s22 / s26 traversals): W = 8 3-5 % / 6-12 % faster than 32, W = 4 alike
    template <int NT> void pull_tiles_dense(const BfsTiles &Q, const BfsView &B, long long nTRl, cudaStream_t s) {
        const int W = getenv("TSMV_PULL_W") ? atoi(getenv("TSMV_PULL_W")) : 8;
        if (W == 16) k_pull_sub<NT, 16><<<grid_for(nTRl * 16), 256, 0, s>>>(Q, B, nTRl);
        else if (W == 8) k_pull_sub<NT, 8><<<grid_for(nTRl * 8), 256, 0, s>>>(Q, B, nTRl);
        else if (W == 4) k_pull_sub<NT, 4><<<grid_for(nTRl * 4), 256, 0, s>>>(Q, B, nTRl);
        else k_pull<NT, false><<<grid_for(nTRl * 32), 256, 0, s>>>(Q, B, nTRl);
    }

    template <int NT> void expand(int dir, bool wide) {
        BfsView B = view();
        BfsTiles P = bfs_tiles(c->P), Q = bfs_tiles(*c->Q);
        if (dir == TSMV_DIR_PUSH_CSC) {
            const int bulk_ok = getenv("TSMV_BFS_NO_BULK") ? 0 : 1;
            k_push<NT, true><<<c->expand_blocks, 256, 0, st>>>(P, lists_view(c), c->counters.as<Counters>(), B,
                                                               bulk_ok);
            if (bulk_ok) k_bulk_fix<<<grid_for((c->m + 31) / 32), 256, 0, st>>>(c->counters.as<Counters>(), B);
        } else if (dir == TSMV_DIR_PUSH_CSR) {
            k_push<NT, false><<<c->expand_blocks, 256, 0, st>>>(P, lists_view(c), c->counters.as<Counters>(), B, 0);
            if (Q.T) k_push_csr<NT><<<grid_for(Q.T), 256, 0, st>>>(Q, B);
        } else {
            long long nTRl = (c->m + NT - 1) / NT;
            if (wide) {
                k_pull<NT, true><<<grid_for(nTRl), 256, 0, st>>>(Q, B, nTRl);
                k_pull_side<NT, true><<<grid_for((c->m + 31) / 32), 256, 0, st>>>(Q, B);
            } else {
                // the tile part and the side part of a dense pull level are independent
                // (both claim new vertices with atomics on V): the side kernel runs on
                // the context's second stream, concurrently with the tile kernel
                // (one launch for both parts, tile blocks first, measured 1.4x slower)
                if (c->aux_stream) {
                    TSMV_CUDA(cudaEventRecord(c->ev_fork, st));
                    TSMV_CUDA(cudaStreamWaitEvent(c->aux_stream, c->ev_fork, 0));
                    pull_side_dense<NT>(Q, B, c->aux_stream);
                    TSMV_CUDA(cudaEventRecord(c->ev_join, c->aux_stream));
                    pull_tiles_dense<NT>(Q, B, nTRl, st);
                    TSMV_CUDA(cudaStreamWaitEvent(st, c->ev_join, 0));
                } else {
                    pull_tiles_dense<NT>(Q, B, nTRl, st);
                    pull_side_dense<NT>(Q, B, st);
                }
            }
        }
        TSMV_CUDA(cudaGetLastError());
    }

    // lists = false: statistics only (|F|, m_f, sum indeg, work totals), for the
    // hybrid driver, whose next push level rebuilds its lists inside the
    // persistent kernel
    void do_fscan(const uint32_t *F, uint32_t *Fclear, bool lists = true, bool lite = false) {
        switch (c->nt) {
            case 16: fscan<16>(F, Fclear, lists, lite); break;
            case 32: fscan<32>(F, Fclear, lists); break;
            default: fscan<64>(F, Fclear, lists); break;
        }
    }
    // wide: late Pull-CSC level (few unvisited edges left), see k_pull
    void do_expand(int dir, bool wide = false) {
        switch (c->nt) {
            case 16: expand<16>(dir, wide); break;
            case 32: expand<32>(dir, wide); break;
            default: expand<64>(dir, wide); break;
        }
    }
    void init(long long source) {
        BfsView B = view();
        k_bfs_init<<<grid_for(std::max<long long>(NW, c->m)), 256, 0, st>>>(B, NW, source);
        TSMV_CUDA(cudaGetLastError());
    }
};

// Host-run pull levels take the wide form (thread per visited word, serial over
// the word's unvisited vertices) only while the unvisited vertices' in-edges are
// few: mu * bfs_wide_mult() < nnz.  r2 used 4, which put R-MAT s26's big pull
// level (mu ~ 95 M of 2.1 G after its frontier) on the wide form: 2.3-3.2 ms
// there against 1.0 ms on the dense kernels (measured: 64).  The distributed
// level loops use the same rule (dist.WIDE_MULT).
long long bfs_wide_mult() {
    static const long long m = getenv("TSMV_BFS_WIDE_MULT") ? atoll(getenv("TSMV_BFS_WIDE_MULT")) : 64;
    return m;
}

// global out-degrees: set for a distributed context (communicator or
// tsmv_bfs_dist_set_degrees); a one-rank context's own column counts are global
static const int *out_degrees(const tsmv_ctx *c) {
    return c->outdeg_g.p ? c->outdeg_g.as<int>() : c->outdeg.as<int>();
}

// this rank's words of the frontier bitmap and its statistics shares (dstats)
static void owned_stats(tsmv_ctx *c, const uint32_t *F, cudaStream_t st) {
    c->dstats.ensure(4 * 8);
    TSMV_CUDA(cudaMemsetAsync(c->dstats.p, 0, 4 * 8, st));
    const long long w0 = c->row_begin >> 5, w1 = (c->row_begin + c->m + 31) >> 5;
    if (w1 > w0)
        k_owned_stats<<<grid_for(w1 - w0, 256, c->sm_count * 8), 256, 0, st>>>(F, w0, w1, c->row_begin, out_degrees(c),
                                                         c->indeg.as<int>(), c->dstats.as<unsigned long long>());
    TSMV_CUDA(cudaGetLastError());
}

int choose_dir(const tsmv_options &o, long long n, long long fsize, long long mf, long long mu, long long fprev) {
    if (o.force_dir != TSMV_DIR_AUTO) return o.force_dir;
    // reading R9: Beamer-style edge test for pull, then the paper's 0.01 density rule;
    // R9': Beamer's alpha on explosive levels (frontier grew burst_growth x)
    const double alpha = burst_alpha(o.pull_alpha, o.pull_alpha_burst, o.burst_growth, fsize, fprev);
    if ((double)mf > (double)mu / alpha) return TSMV_DIR_PULL_CSC;
    if ((double)fsize / (double)n >= o.push_csr_density) return TSMV_DIR_PUSH_CSR;
    return TSMV_DIR_PUSH_CSC;
}

}  // namespace tsmv

using namespace tsmv;

static void bfs_check(tsmv_ctx *c) {
    TSMV_REQUIRE(c->bfs_built, "tsmv_bfs: context built without BFS structures (square A and build_bfs=1 needed)");
    TSMV_REQUIRE(!c->bfs_block2d, "tsmv_bfs: a 2D block context (build_bfs = 2) serves tsmv_bfs2d_expand only");
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

// level_ms[L] = time from level L's expansion decision to level L+1's (the last
// level: to the end of the traversal), from the stamps in c->bfs_tlv
static void level_times(tsmv_ctx *c, tsmv_bfs_stats *stats, long long nl, bool has_end) {
    std::vector<unsigned long long> t(nl + 1, 0);
    TSMV_CUDA(cudaMemcpy(t.data(), c->bfs_tlv.p, (nl + (has_end ? 1 : 0)) * 8, cudaMemcpyDeviceToHost));
    for (long long L = 0; L < nl; ++L)
        stats->level_ms[L] = (L + 1 < nl || has_end) && t[L + 1] >= t[L] ? (float)((t[L + 1] - t[L]) * 1e-6) : 0.f;
}

// Distributed TileBFS of a context with its own communicator:
// Alg 3's level loop on every rank, one exchange per level.  The
// frontier F and the visited bitmap V are replicated (n bits); each rank expands
// the level into its OWNED rows with the level kernels (Push-CSC / Push-CSR /
// Pull-CSC over its row block; the push lists are built from the replicated
// frontier on push levels only), computes the statistics shares of its owned
// new vertices (count, sum of global out-degrees, sum of in-degrees: O(n / P)),
// and one NCCL group broadcasts the owned frontier words in place and
// all-gathers the shares; every rank sums the same shares, hence takes the same
// direction decision and stops at the same level.  One host synchronisation per
// level (the statistics choose the kernels).  Nothing per level is O(n) except
// the OR of the frontier into V (n / 32 words) and the clearing of the old one.
static void bfs_distributed(tsmv_ctx *c, int64_t source, tsmv_bfs_stats *stats, cudaStream_t st) {
    ensure_lists(c, c->n);
    BfsRunner R{c, st, (long long)(c->V.bytes / 4)};
    unsigned long long *tlv = c->bfs_tlv.as<unsigned long long>();
    const int P = c->opt.nranks;
    c->dstats_all.ensure((size_t)P * 4 * 8);
    std::vector<unsigned long long> sh((size_t)P * 4);
    c->fcur = 0;
    c->bfs_level = 0;
    TSMV_CUDA(cudaEventRecord(c->ev0, st));
    TSMV_CUDA(cudaMemsetAsync(c->F1.p, 0, c->F1.bytes, st));
    R.init(source);
    long long fsize = 1, mf = 0, mu = c->nnz_global;
    {
        int od = 0, id = 0;
        TSMV_CUDA(cudaMemcpyAsync(&od, c->outdeg_g.as<int>() + source, 4, cudaMemcpyDeviceToHost, st));
        TSMV_CUDA(cudaMemcpyAsync(&id, c->indeg_g.as<int>() + source, 4, cudaMemcpyDeviceToHost, st));
        TSMV_CUDA(cudaStreamSynchronize(st));
        mf = od;
        mu -= id;
    }
    long long reached = 0, edges = 0;
    long long L = 0, fprev = 0;
    while (fsize > 0) {
        const int dir = choose_dir(c->opt, c->n, fsize, mf, mu, fprev);
        fprev = fsize;
        if (L < TSMV_MAX_LEVELS) {
            if (stats) {
                stats->dir_per_level[L] = dir;
                stats->frontier_per_level[L] = fsize;
            }
            k_stamp<<<1, 1, 0, st>>>(tlv + L);
        }
        reached += fsize;
        edges += mf;
        c->bfs_level = (int)L;
        uint32_t *Fcur = (c->fcur == 0 ? c->F0 : c->F1).as<uint32_t>();
        uint32_t *Fnext = (c->fcur == 0 ? c->F1 : c->F0).as<uint32_t>();
        if (dir != TSMV_DIR_PULL_CSC) R.do_fscan(Fcur, nullptr);  // push lists of the replicated frontier
        R.do_expand(dir, dir == TSMV_DIR_PULL_CSC && mu * bfs_wide_mult() < c->nnz_global);
        owned_stats(c, Fnext, st);
        comm_exchange_frontier(c, Fnext, c->V.as<uint32_t>(), (c->n + 31) / 32, c->dstats.p, c->dstats_all.p, st);
        TSMV_CUDA(cudaMemsetAsync(Fcur, 0, ((c->n + 63) / 64) * 8, st));
        TSMV_CUDA(cudaMemcpyAsync(sh.data(), c->dstats_all.p, sh.size() * 8, cudaMemcpyDeviceToHost, st));
        TSMV_CUDA(cudaStreamSynchronize(st));
        fsize = mf = 0;
        long long din = 0;
        for (int p = 0; p < P; ++p) {
            fsize += (long long)sh[p * 4];
            mf += (long long)sh[p * 4 + 1];
            din += (long long)sh[p * 4 + 2];
        }
        mu -= din;
        c->fcur ^= 1;
        ++L;
    }
    if (L <= TSMV_MAX_LEVELS) k_stamp<<<1, 1, 0, st>>>(tlv + L);
    TSMV_CUDA(cudaEventRecord(c->ev1, st));
    TSMV_CUDA(cudaMemsetAsync(c->F0.p, 0, c->F0.bytes, st));
    TSMV_CUDA(cudaMemsetAsync(c->F1.p, 0, c->F1.bytes, st));
    TSMV_CUDA(cudaStreamSynchronize(st));
    c->bfs_last_levels = L;
    if (stats) {
        float ms = 0;
        TSMV_CUDA(cudaEventElapsedTime(&ms, c->ev0, c->ev1));
        stats->nlevels = (int32_t)std::min<long long>(L, INT32_MAX);
        if (L > 0) level_times(c, stats, std::min<long long>(L, TSMV_MAX_LEVELS), L <= TSMV_MAX_LEVELS);
        stats->reached = reached;
        stats->edges_traversed = edges;
        stats->ms = ms;
    }
}

extern "C" tsmv_status tsmv_bfs(tsmv_ctx *c, int64_t source, int32_t *levels, tsmv_bfs_stats *stats,
                                void *cuda_stream) {
    try {
        TSMV_REQUIRE(c != nullptr && levels != nullptr, "tsmv_bfs: NULL argument");
        bfs_check(c);
        if (has_comm(c)) {
            TSMV_REQUIRE(source >= 0 && source < c->n, "tsmv_bfs: source %lld out of range", (long long)source);
            TSMV_CUDA(cudaSetDevice(c->device));
            cudaStream_t st = (cudaStream_t)cuda_stream;
            bool host_levels;
            bfs_prepare_levels(c, levels, host_levels);
            bfs_distributed(c, source, stats, st);
            if (host_levels) {
                TSMV_CUDA(cudaMemcpyAsync(levels, c->levels_dev, c->m * 4, cudaMemcpyDeviceToHost, st));
                TSMV_CUDA(cudaStreamSynchronize(st));
            }
            return TSMV_OK;
        }
        TSMV_REQUIRE(c->opt.nranks == 1,
                     "tsmv_bfs: a distributed context needs its own communicator (tsmv_options.nccl_unique_id) "
                     "or the tsmv_bfs_dist_* calls");
        TSMV_REQUIRE(source >= 0 && source < c->n, "tsmv_bfs: source %lld out of range", (long long)source);
        TSMV_CUDA(cudaSetDevice(c->device));
        cudaStream_t st = (cudaStream_t)cuda_stream;
        bool host_levels;
        bfs_prepare_levels(c, levels, host_levels);
        ensure_lists(c, c->n);
        if (!getenv("TSMV_BFS_HOSTLOOP")) {
            // Hybrid: push levels run inside the fused persistent kernel
            // (no host round trip per level); a Pull-CSC level hands back to the host,
            // which runs it with the high-occupancy per-level kernels, then resumes.
            const bool stop_on_pull = !getenv("TSMV_BFS_FUSED_ONLY");
            TSMV_CUDA(cudaEventRecord(c->ev0, st));
            uint32_t *Fa = c->F0.as<uint32_t>(), *Fb = c->F1.as<uint32_t>();
            long long level = 0, mu = c->nnz, reached = 0, edges = 0;
            long long fprev = 0;  // |F| of the level before `level` (R9')
            bool resume = false;
            BfsRunner R{c, st, (long long)(c->V.bytes / 4)};
            const long long maxlv = getenv("TSMV_BFS_MAXLV") ? atoll(getenv("TSMV_BFS_MAXLV")) : (1ll << 40);
            unsigned long long *tlv = c->bfs_tlv.as<unsigned long long>();
            const bool tline = getenv("TSMV_BFS_TIMELINE") != nullptr;  // dev aid: host pull level kernel times
            const long long wide_mult = bfs_wide_mult();
            // resuming right behind a host pull level pays the persistent kernel's count
            // phase instead of the statistics pass and a host round trip: only while
            // that bitmap scan is short (<= 4 nt-segments per thread: R-MAT s22 yes,
            // s26 no, where consecutive dense pull levels stay on the host as in r2)
            const bool host_decide = getenv("TSMV_BFS_HOST_DECIDE") != nullptr ||
                                     (c->nTC > 4ll * c->bfs_blocks * 512 && !getenv("TSMV_BFS_RESUME_BEHIND"));
            while (true) {
                long long L, mu2, r2, e2;
                int cur;
                long long fexp = 0;  // stopped: |F| of the level the host expands next
                const bool stopped = bfs_fused_launch(c, source, st, resume, level, Fa, Fb, mu, reached, edges,
                                                      stop_on_pull, maxlv, L, mu2, r2, e2, cur, fprev, fexp);
                if (getenv("TSMV_BFS_PHASES")) {
                    long long fl = 0;
                    if (c->lslots.p) {
                        TSMV_CUDA(cudaMemcpy(&fl, c->lslots.as<long long>() + 15, 8, cudaMemcpyDeviceToHost));
                        TSMV_CUDA(cudaMemset(c->lslots.as<long long>() + 12, 0, 32));
                    }
                    fprintf(stderr, "[bfs fused] levels %lld..%lld: count %.3f ms, lists %.3f ms, expand %.3f ms"
                            " (list-prof builds: CTA0 expand / slowest CTA / CTA0 flush %.3f ms)\n",
                            level, L, c->hcnt->Wt * 1e-6, c->hcnt->nLs * 1e-6, c->hcnt->Ws * 1e-6, fl * 1e-6);
                }
                if (cur) std::swap(Fa, Fb);  // Fa = bitmap of the current frontier
                level = L;
                mu = mu2;
                reached = r2;
                edges = e2;
                if (!stopped) break;
                if (c->bfs_stop_kind == 2) {
                    // a heavy bulk Push-CSC level whose lists the kernel built: the
                    // high-occupancy k_push / k_bulk_fix run it, then the kernel resumes
                    c->bfs_level = (int)level;
                    c->fcur = (Fa == c->F0.as<uint32_t>()) ? 0 : 1;
                    R.do_expand(TSMV_DIR_PUSH_CSC);
                    std::swap(Fa, Fb);
                    ++level;
                    fprev = fexp;
                    resume = true;
                    continue;
                }
                if (!host_decide) {
                    // the level the kernel stopped at is a pull level: the host kernels run
                    // it and the persistent kernel is resumed right behind them on the
                    // stream (no host round trip, no statistics pass: the resumed count
                    // phase takes the next frontier's statistics, clears the consumed
                    // bitmap and decides, stopping again for another dense pull level)
                    c->bfs_level = (int)level;
                    c->fcur = (Fa == c->F0.as<uint32_t>()) ? 0 : 1;
                    R.do_expand(TSMV_DIR_PULL_CSC, mu * wide_mult < c->nnz);
                    std::swap(Fa, Fb);
                    ++level;
                    fprev = fexp;
                    resume = true;
                    continue;
                }
                // (r2) pull levels on the host path until the rule turns back to push
                while (true) {
                    c->bfs_level = (int)level;
                    c->fcur = (Fa == c->F0.as<uint32_t>()) ? 0 : 1;
                    unsigned long long *tl = tline ? c->bfs_tlv.as<unsigned long long>() + TSMV_MAX_LEVELS - 8 : nullptr;
                    if (tl) k_stamp<<<1, 1, 0, st>>>(tl + 0);
                    // (statistics taken at discovery in the pull kernels: the tile part's
                    // warps then wait on every claim, measured 1.4x slower than this pass)
                    R.do_expand(TSMV_DIR_PULL_CSC, mu * wide_mult < c->nnz);
                    if (tl) k_stamp<<<1, 1, 0, st>>>(tl + 1);
                    R.do_fscan(Fb, Fa, false, true);  // next frontier |F|, m_f, din; clears Fa
                    if (tl) k_stamp<<<1, 1, 0, st>>>(tl + 2);
                    TSMV_CUDA(cudaStreamSynchronize(st));
                    if (tl) {
                        unsigned long long t[3];
                        TSMV_CUDA(cudaMemcpy(t, tl, 24, cudaMemcpyDeviceToHost));
                        fprintf(stderr, "[bfs host pull] level %lld: expand %.1f us, stats %.1f us\n", level,
                                (t[1] - t[0]) * 1e-3, (t[2] - t[1]) * 1e-3);
                    }
                    volatile Counters *h = c->hcnt;
                    const long long fsize = h->fsize, mf = h->mf, din = h->din;
                    std::swap(Fa, Fb);
                    ++level;
                    if (fsize == 0 || level >= maxlv) break;
                    const int dir = choose_dir(c->opt, c->n, fsize, mf, mu - din, fexp);
                    fprev = fexp;  // the kernel re-decides `level` from here when it resumes
                    // resume the fused kernel at `level` for push levels and for the late
                    // (wide) pull levels, which it runs in place without host round trips
                    if (dir != TSMV_DIR_PULL_CSC || (!getenv("TSMV_BFS_HOST_WIDE") && (mu - din) * 4 < c->nnz &&
                                                     mu - din <= bfs_wide_cap(c, true)))
                        break;
                    mu -= din;
                    reached += fsize;
                    edges += mf;
                    fexp = fsize;
                    if (level < TSMV_MAX_LEVELS)
                        k_level_rec<<<1, 1, 0, st>>>(c->bfs_dirs.as<int>() + level, c->bfs_front.as<long long>() + level,
                                                     tlv + level, dir, fsize);
                }
                if (c->hcnt->fsize == 0 || level >= maxlv) break;
                resume = true;
            }
            if (level <= TSMV_MAX_LEVELS) k_stamp<<<1, 1, 0, st>>>(tlv + level);
            TSMV_CUDA(cudaEventRecord(c->ev1, st));
            if (host_levels) TSMV_CUDA(cudaMemcpyAsync(levels, c->levels_dev, c->m * 4, cudaMemcpyDeviceToHost, st));
            TSMV_CUDA(cudaStreamSynchronize(st));
            c->bfs_last_levels = level;
            if (stats) {
                float ms = 0;
                TSMV_CUDA(cudaEventElapsedTime(&ms, c->ev0, c->ev1));
                const long long nl = std::min<long long>(level, TSMV_MAX_LEVELS);
                if (nl > 0) {
                    TSMV_CUDA(cudaMemcpy(stats->dir_per_level, c->bfs_dirs.p, nl * 4, cudaMemcpyDeviceToHost));
                    TSMV_CUDA(cudaMemcpy(stats->frontier_per_level, c->bfs_front.p, nl * 8, cudaMemcpyDeviceToHost));
                    level_times(c, stats, nl, level <= TSMV_MAX_LEVELS);
                }
                stats->nlevels = (int32_t)std::min<long long>(level, INT32_MAX);
                stats->reached = reached;
                stats->edges_traversed = edges;
                stats->ms = ms;
            }
            return TSMV_OK;
        }
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
        long long reached = 0, edges = 0, fprev = 0;
        int L = 0;
        if (stats) stats->nlevels = 0;
        unsigned long long *tlv = c->bfs_tlv.as<unsigned long long>();
        while (fsize > 0) {
            int dir = choose_dir(c->opt, c->n, fsize, mf, mu, fprev);
            fprev = fsize;
            if (stats && L < TSMV_MAX_LEVELS) {
                stats->dir_per_level[L] = dir;
                stats->frontier_per_level[L] = fsize;
            }
            if (L < TSMV_MAX_LEVELS) k_stamp<<<1, 1, 0, st>>>(tlv + L);
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
        if (L <= TSMV_MAX_LEVELS) k_stamp<<<1, 1, 0, st>>>(tlv + L);
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
            if (L > 0) level_times(c, stats, std::min<long long>(L, TSMV_MAX_LEVELS), L <= TSMV_MAX_LEVELS);
            stats->reached = reached;
            stats->edges_traversed = edges;
            stats->ms = ms;
        }
        return TSMV_OK;
    } catch (const Err &e) {
        return e.st;
    }
}

// Chunk list (vertex << 24 | chunk of 256 entries) of the side rows of Q with
// more than 32 entries (power-law hubs), built once per context; used by the
// parents and multi-source BFS kernels.
void tsmv::heavy_side_chunks(tsmv_ctx *c, cudaStream_t st) {
    if (c->par_chunks.p) return;
    DevBuf cnt, off;
    cnt.alloc(std::max<long long>(c->m, 1) * 4);
    k_par_chunk_count<<<grid_for(c->m), 256, 0, st>>>(c->Q->sptr.as<long long>(), c->m, cnt.as<int>());
    std::vector<int> hc(c->m);
    TSMV_CUDA(cudaMemcpyAsync(hc.data(), cnt.p, c->m * 4, cudaMemcpyDeviceToHost, st));
    TSMV_CUDA(cudaStreamSynchronize(st));
    std::vector<long long> ho(c->m);
    long long tot = 0;
    for (long long v = 0; v < c->m; ++v) {
        ho[v] = tot;
        tot += hc[v];
    }
    off.alloc(std::max<long long>(c->m, 1) * 8);
    TSMV_CUDA(cudaMemcpyAsync(off.p, ho.data(), c->m * 8, cudaMemcpyHostToDevice, st));
    c->par_chunks.alloc(std::max<long long>(tot, 1) * 8);
    k_par_chunk_fill<<<grid_for(c->m), 256, 0, st>>>(c->Q->sptr.as<long long>(), c->m, off.as<long long>(),
                                                     cnt.as<int>(), c->par_chunks.as<long long>());
    TSMV_CUDA(cudaStreamSynchronize(st));
    c->par_nchunks = tot;
}

extern "C" tsmv_status tsmv_bfs_parents(tsmv_ctx *c, const int32_t *levels, int32_t *parents, void *cuda_stream) {
    try {
        TSMV_REQUIRE(c != nullptr && levels != nullptr && parents != nullptr, "tsmv_bfs_parents: NULL argument");
        bfs_check(c);
        TSMV_REQUIRE(c->opt.nranks == 1, "tsmv_bfs_parents: single-GPU contexts only");
        TSMV_REQUIRE(is_device_ptr(levels) && is_device_ptr(parents),
                     "tsmv_bfs_parents: levels and parents must be device memory");
        TSMV_CUDA(cudaSetDevice(c->device));
        cudaStream_t st = (cudaStream_t)cuda_stream;
        BfsTiles Q = bfs_tiles(*c->Q);
        const int grid = grid_for(c->m * 32);
        if (c->nt == 16) {
            const long long nTR = (c->m + 15) / 16;
            k_parents_tiles16<<<grid_for(nTR * 32), 256, 0, st>>>(Q, levels, parents, c->m, nTR);
            k_parents_side<16, false><<<grid_for(c->m), 256, 0, st>>>(Q, levels, parents, c->m);
            heavy_side_chunks(c, st);
            if (c->par_nchunks)
                k_parents_chunks<16><<<grid_for(c->par_nchunks * 32), 256, 0, st>>>(
                    Q, levels, parents, c->par_chunks.as<long long>(), c->par_nchunks);
            k_parents_fix<<<grid_for(c->m), 256, 0, st>>>(parents, c->m);
        } else if (c->nt == 32) k_parents<32><<<grid, 256, 0, st>>>(Q, levels, parents, c->m);
        else k_parents<64><<<grid, 256, 0, st>>>(Q, levels, parents, c->m);
        TSMV_CUDA(cudaGetLastError());
        return TSMV_OK;
    } catch (const Err &e) {
        return e.st;
    }
}

// ----------------------------------------------------------------- distributed primitives
extern "C" int64_t tsmv_owned_words(const tsmv_ctx *c) { return c ? (c->m + 31) / 32 : 0; }

extern "C" tsmv_status tsmv_bfs_dist_set_degrees(tsmv_ctx *c, const int32_t *outdeg_global) {
    try {
        TSMV_REQUIRE(c && outdeg_global, "tsmv_bfs_dist_set_degrees: NULL argument");
        TSMV_CUDA(cudaSetDevice(c->device));
        c->outdeg_g.alloc(((std::max<int64_t>(c->n, 1) + 63) / 64 * 64) * 4);
        TSMV_CUDA(cudaMemset(c->outdeg_g.p, 0, c->outdeg_g.bytes));
        TSMV_CUDA(cudaMemcpy(c->outdeg_g.p, outdeg_global, c->n * 4, cudaMemcpyDefault));
        return TSMV_OK;
    } catch (const Err &e) {
        return e.st;
    }
}

static void dist_out(tsmv_ctx *c, int64_t *out_stats, cudaStream_t st) {
    if (is_device_ptr(out_stats)) {
        // device statistics: no synchronisation (the caller reduces them on the device)
        k_dist_stats2<<<1, 1, 0, st>>>(c->dstats.as<unsigned long long>(), c->mu_dev.as<long long>(), out_stats);
        TSMV_CUDA(cudaGetLastError());
        return;
    }
    unsigned long long h[4];
    TSMV_CUDA(cudaMemcpyAsync(h, c->dstats.p, 32, cudaMemcpyDeviceToHost, st));
    TSMV_CUDA(cudaStreamSynchronize(st));
    c->m_u_local -= (long long)h[2];
    TSMV_CUDA(cudaMemcpyAsync(c->mu_dev.p, &c->m_u_local, 8, cudaMemcpyHostToDevice, st));
    TSMV_CUDA(cudaStreamSynchronize(st));
    out_stats[0] = (long long)h[0];
    out_stats[1] = (long long)h[1];
    out_stats[2] = c->m_u_local;
}

extern "C" tsmv_status tsmv_bfs_dist_begin(tsmv_ctx *c, int64_t source, int32_t *levels, int64_t *out_stats,
                                           void *cuda_stream) {
    try {
        TSMV_REQUIRE(c && levels && out_stats, "tsmv_bfs_dist_begin: NULL argument");
        bfs_check(c);
        TSMV_REQUIRE(source >= 0 && source < c->n, "tsmv_bfs_dist_begin: source out of range");
        TSMV_REQUIRE(is_device_ptr(levels), "tsmv_bfs_dist_begin: levels must be device memory");
        TSMV_REQUIRE(c->outdeg_g.p != nullptr || c->opt.nranks == 1,
                     "tsmv_bfs_dist_begin: global out-degrees not set (tsmv_bfs_dist_set_degrees)");
        TSMV_CUDA(cudaSetDevice(c->device));
        cudaStream_t st = (cudaStream_t)cuda_stream;
        c->levels_dev = levels;
        ensure_lists(c, c->n);
        BfsRunner R{c, st, (long long)(c->V.bytes / 4)};
        c->fcur = 0;
        c->bfs_level = 0;
        TSMV_CUDA(cudaMemsetAsync(c->F1.p, 0, c->F1.bytes, st));
        R.init(source);
        c->dstats.ensure(32);
        k_source_stats<<<1, 1, 0, st>>>(source, c->row_begin, c->m, out_degrees(c), c->indeg.as<int>(),
                                       c->dstats.as<unsigned long long>());
        TSMV_CUDA(cudaGetLastError());
        c->m_u_local = c->nnz;
        c->mu_dev.ensure(8);
        TSMV_CUDA(cudaMemcpyAsync(c->mu_dev.p, &c->m_u_local, 8, cudaMemcpyHostToDevice, st));
        dist_out(c, out_stats, st);
        return TSMV_OK;
    } catch (const Err &e) {
        return e.st;
    }
}

extern "C" tsmv_status tsmv_bfs_dist_expand(tsmv_ctx *c, int32_t dir, uint32_t *owned_words_out, void *cuda_stream) {
    try {
        TSMV_REQUIRE(c && owned_words_out, "tsmv_bfs_dist_expand: NULL argument");
        const bool wide = (dir & TSMV_DIST_WIDE) != 0;
        dir &= ~TSMV_DIST_WIDE;
        TSMV_REQUIRE(dir >= 1 && dir <= 3, "tsmv_bfs_dist_expand: dir must be concrete (1..3)");
        TSMV_REQUIRE(c->levels_dev != nullptr, "tsmv_bfs_dist_expand: no traversal begun (tsmv_bfs_dist_begin)");
        TSMV_CUDA(cudaSetDevice(c->device));
        cudaStream_t st = (cudaStream_t)cuda_stream;
        BfsRunner R{c, st, (long long)(c->V.bytes / 4)};
        uint32_t *Fcur = (c->fcur == 0 ? c->F0 : c->F1).as<uint32_t>();
        uint32_t *Fnext = (c->fcur == 0 ? c->F1 : c->F0).as<uint32_t>();
        if (dir != TSMV_DIR_PULL_CSC) R.do_fscan(Fcur, nullptr);  // push lists of the replicated frontier
        R.do_expand(dir, wide && dir == TSMV_DIR_PULL_CSC);
        owned_stats(c, Fnext, st);
        TSMV_CUDA(cudaMemcpyAsync(owned_words_out, Fnext + (c->row_begin >> 5), tsmv_owned_words(c) * 4,
                                  cudaMemcpyDeviceToDevice, st));
        return TSMV_OK;
    } catch (const Err &e) {
        return e.st;
    }
}

// 2D block level (bfs2d.cu's sequence, include/tsmv.h): the level kernels of the
// row-block path on caller-provided row bitmaps (visited / next over R_i) and the
// column frontier of C_j staged in F0 (zero-padded to whole 16-byte vectors)
extern "C" tsmv_status tsmv_bfs2d_expand(tsmv_ctx *c, int32_t dir, const uint32_t *x_words, const uint32_t *row_new,
                                         uint32_t *visited_rows, uint32_t *next_words, int32_t *levels_rows,
                                         int32_t level, void *cuda_stream) {
    try {
        TSMV_REQUIRE(c && x_words && visited_rows && next_words && levels_rows, "tsmv_bfs2d_expand: NULL argument");
        TSMV_REQUIRE(c->bfs_built && c->bfs_block2d, "tsmv_bfs2d_expand: context not built with build_bfs = 2");
        const bool wide = (dir & TSMV_DIST_WIDE) != 0;
        dir &= ~TSMV_DIST_WIDE;
        TSMV_REQUIRE(dir >= 1 && dir <= 3, "tsmv_bfs2d_expand: dir must be concrete (1..3)");
        TSMV_REQUIRE(is_device_ptr(x_words) && (!row_new || is_device_ptr(row_new)) && is_device_ptr(visited_rows) &&
                         is_device_ptr(next_words) && is_device_ptr(levels_rows),
                     "tsmv_bfs2d_expand: device memory expected");
        TSMV_CUDA(cudaSetDevice(c->device));
        cudaStream_t st = (cudaStream_t)cuda_stream;
        const long long nwr = (c->m + 31) / 32, nwx = (c->n + 31) / 32, nwpad = (long long)(c->V.bytes / 4);
        uint32_t *F = c->F0.as<uint32_t>();
        // one launch: visited_rows |= row_new, next_words = 0, F0 = x (zero-padded)
        k_level2d_prep<<<grid_for(std::max(nwr, nwpad)), 256, 0, st>>>(visited_rows, row_new, next_words, nwr, F,
                                                                        x_words, nwx, nwpad);
        TSMV_CUDA(cudaGetLastError());
        ensure_lists(c, c->n);
        BfsView B;
        B.V = visited_rows;
        B.F = F;
        B.Fn = next_words;
        B.levels = levels_rows;
        B.row_begin = 0;
        B.m_local = c->m;
        B.n = c->n;
        B.level = level;
        BfsRunner R{c, st, nwpad};
        R.ov = &B;
        if (dir != TSMV_DIR_PULL_CSC) R.do_fscan(F, nullptr);
        R.do_expand(dir, wide && dir == TSMV_DIR_PULL_CSC);
        return TSMV_OK;
    } catch (const Err &e) {
        return e.st;
    }
}

extern "C" tsmv_status tsmv_bfs_dist_merge(tsmv_ctx *c, const uint32_t *gathered, int64_t stride_words,
                                           int64_t *out_stats, void *cuda_stream) {
    try {
        TSMV_REQUIRE(c && out_stats, "tsmv_bfs_dist_merge: NULL argument");
        bfs_check(c);
        TSMV_REQUIRE(c->levels_dev != nullptr, "tsmv_bfs_dist_merge: no traversal begun (tsmv_bfs_dist_begin)");
        if (c->opt.nranks > 1) {
            long long need = 0;
            for (int p = 0; p < c->opt.nranks; ++p)
                need = std::max<long long>(need, (c->row_splits[p + 1] - c->row_splits[p] + 31) / 32);
            TSMV_REQUIRE(stride_words >= need, "tsmv_bfs_dist_merge: stride_words %lld < largest owned segment %lld",
                         (long long)stride_words, need);
            TSMV_REQUIRE(is_device_ptr(gathered), "tsmv_bfs_dist_merge: gathered must be device memory");
        }
        TSMV_CUDA(cudaSetDevice(c->device));
        cudaStream_t st = (cudaStream_t)cuda_stream;
        uint32_t *Fcur = (c->fcur == 0 ? c->F0 : c->F1).as<uint32_t>();
        uint32_t *Fnext = (c->fcur == 0 ? c->F1 : c->F0).as<uint32_t>();
        if (c->opt.nranks > 1) {
            TSMV_REQUIRE(gathered != nullptr, "tsmv_bfs_dist_merge: NULL gathered");
            k_merge<<<grid_for(stride_words), 256, 0, st>>>(gathered, stride_words, c->opt.nranks,
                                                            c->splits_dev.as<long long>(), c->opt.rank, Fnext,
                                                            c->V.as<uint32_t>());
            TSMV_CUDA(cudaGetLastError());
        }
        TSMV_CUDA(cudaMemsetAsync(Fcur, 0, ((c->n + 63) / 64) * 8, st));
        c->fcur ^= 1;
        c->bfs_level += 1;
        dist_out(c, out_stats, st);
        return TSMV_OK;
    } catch (const Err &e) {
        return e.st;
    }
}

extern "C" int32_t tsmv_choose_dir(const tsmv_options *o, int64_t n, int64_t frontier, int64_t m_f, int64_t m_u,
                                   int64_t prev_frontier) {
    tsmv_options d;
    if (!o) {
        tsmv_default_options(&d);
        o = &d;
    }
    return choose_dir(*o, n, frontier, m_f, m_u, prev_frontier);
}
