// device.cuh -- device helpers shared by the SpMSpV and TileBFS kernels:
// single-pass decoupled look-back scan, dynamic block ids, list/chunk writers,
// and the chunk -> list-entry window search of the load-balanced expand kernels.
#pragma once
#include "common.cuh"
#include <cub/block/block_scan.cuh>

namespace tsmv {

struct Quad {
    long long v[4];
};
struct QuadSum {
    __device__ __forceinline__ Quad operator()(const Quad &a, const Quad &b) const {
        Quad r;
#pragma unroll
        for (int i = 0; i < 4; ++i) r.v[i] = a.v[i] + b.v[i];
        return r;
    }
};

__device__ __forceinline__ unsigned ld_status(const LBDesc<4> *d) {
    return *(volatile const unsigned *)&d->status;
}
template <int K> __device__ __forceinline__ unsigned ld_status_k(const LBDesc<K> *d) {
    return *(volatile const unsigned *)&d->status;
}

// Decoupled look-back (one thread per block).  `agg` = this block's aggregate,
// returns the exclusive prefix of all blocks before `bid`.  Blocks must obtain
// `bid` in launch order (dynamic ids) so that predecessors are resident.
template <int K>
__device__ void lookback(LBDesc<K> *desc, unsigned bid, unsigned epoch, const long long *agg, long long *excl) {
    const unsigned ep = (epoch & 0x3fffffffu) << 2;
    LBDesc<K> *me = desc + bid;
    if (bid == 0) {
#pragma unroll
        for (int i = 0; i < K; ++i) {
            ((volatile long long *)me->inc)[i] = agg[i];
            excl[i] = 0;
        }
        __threadfence();
        *(volatile unsigned *)&me->status = ep | 2u;
        return;
    }
#pragma unroll
    for (int i = 0; i < K; ++i) ((volatile long long *)me->agg)[i] = agg[i];
    __threadfence();
    *(volatile unsigned *)&me->status = ep | 1u;
    long long acc[K];
#pragma unroll
    for (int i = 0; i < K; ++i) acc[i] = 0;
    int p = (int)bid - 1;
    while (true) {
        unsigned s = ld_status_k<K>(desc + p);
        if ((s & ~3u) != ep || (s & 3u) == 0) continue;
        __threadfence();
        if ((s & 3u) == 2u) {
#pragma unroll
            for (int i = 0; i < K; ++i) acc[i] += ((volatile long long *)desc[p].inc)[i];
            break;
        }
#pragma unroll
        for (int i = 0; i < K; ++i) acc[i] += ((volatile long long *)desc[p].agg)[i];
        --p;
    }
#pragma unroll
    for (int i = 0; i < K; ++i) {
        excl[i] = acc[i];
        ((volatile long long *)me->inc)[i] = acc[i] + agg[i];
    }
    __threadfence();
    *(volatile unsigned *)&me->status = ep | 2u;
}

// Warp-parallel decoupled look-back: called by all 32 lanes of one warp; lane l
// inspects predecessor (window_top - l), so a chain of aggregates is consumed 32
// blocks per L2 round trip.  Same contract as lookback().
template <int K>
__device__ void lookback_warp(LBDesc<K> *desc, unsigned bid, unsigned epoch, const long long *agg, long long *excl,
                              int lane) {
    const unsigned ep = (epoch & 0x3fffffffu) << 2;
    LBDesc<K> *me = desc + bid;
    if (bid == 0) {
        if (lane == 0) {
#pragma unroll
            for (int i = 0; i < K; ++i) ((volatile long long *)me->inc)[i] = agg[i];
            __threadfence();
            *(volatile unsigned *)&me->status = ep | 2u;
        }
#pragma unroll
        for (int i = 0; i < K; ++i) excl[i] = 0;
        return;
    }
    if (lane == 0) {
#pragma unroll
        for (int i = 0; i < K; ++i) ((volatile long long *)me->agg)[i] = agg[i];
        __threadfence();
        *(volatile unsigned *)&me->status = ep | 1u;
    }
    long long acc[K];
#pragma unroll
    for (int i = 0; i < K; ++i) acc[i] = 0;
    long long top = (long long)bid - 1;
    while (true) {
        const long long q = top - lane;
        unsigned s = ep | 2u;  // q < 0: virtual inclusive prefix 0
        if (q >= 0) {
            do {
                s = ld_status_k<K>(desc + q);
            } while ((s & ~3u) != ep || (s & 3u) == 0);
        }
        __syncwarp();
        const unsigned pm = __ballot_sync(0xffffffffu, (s & 3u) == 2u);
        const int first = pm ? __ffs(pm) - 1 : 32;
        __threadfence();
        long long v[K];
#pragma unroll
        for (int i = 0; i < K; ++i) {
            v[i] = 0;
            if (q >= 0 && lane < first) v[i] = ((volatile long long *)desc[q].agg)[i];
            else if (q >= 0 && lane == first) v[i] = ((volatile long long *)desc[q].inc)[i];
        }
#pragma unroll
        for (int i = 0; i < K; ++i) {
#pragma unroll
            for (int o = 16; o > 0; o >>= 1) v[i] += __shfl_xor_sync(0xffffffffu, v[i], o);
            acc[i] += v[i];
        }
        if (first < 32) break;
        top -= 32;
    }
#pragma unroll
    for (int i = 0; i < K; ++i) excl[i] = acc[i];
    if (lane == 0) {
#pragma unroll
        for (int i = 0; i < K; ++i) ((volatile long long *)me->inc)[i] = acc[i] + agg[i];
        __threadfence();
        *(volatile unsigned *)&me->status = ep | 2u;
    }
}

// Exclusive block-wide scan of K int64 values per thread (shuffles + one smem
// pass); register-light replacement for cub::BlockScan of a 4-wide struct, which
// made the fused kernel spill.  tot = block totals (all threads).  Contains
// __syncthreads; every thread of the block must call it.
template <int K, int NTHREADS>
__device__ __forceinline__ void block_scan(const long long *v, long long *ex, long long *tot,
                                           long long (*s)[NTHREADS / 32]) {
    constexpr int NW = NTHREADS / 32;
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
#pragma unroll
    for (int i = 0; i < K; ++i) {
        long long x = v[i];
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const long long y = __shfl_up_sync(0xffffffffu, x, o);
            if (lane >= o) x += y;
        }
        ex[i] = x - v[i];
        if (lane == 31) s[i][wid] = x;
    }
    __syncthreads();
    if (wid == 0) {  // scan the NW warp totals with one warp, in place (exclusive) + total in slot NW-1's place
#pragma unroll
        for (int i = 0; i < K; ++i) {
            const long long w0 = lane < NW ? s[i][lane] : 0;
            long long x = w0;
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                const long long y = __shfl_up_sync(0xffffffffu, x, o);
                if (lane >= o) x += y;
            }
            const long long all = __shfl_sync(0xffffffffu, x, 31);
            if (lane < NW) s[i][lane] = x - w0;
            if (lane == 0) s[i + K][0] = all;
        }
    }
    __syncthreads();
#pragma unroll
    for (int i = 0; i < K; ++i) {
        ex[i] += s[i][wid];
        tot[i] = s[i + K][0];
    }
    __syncthreads();
}

// ------------------------------------------------------------------ grid barrier
// For cooperative (co-resident) launches.  `bar` is a monotonically increasing
// arrival counter; every block tracks the same target sequence from the host-side
// base value of this launch, so nothing has to be reset between launches.
__device__ __forceinline__ unsigned long long ld_acquire_u64(const unsigned long long *p) {
    unsigned long long v;
    asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}

__device__ __forceinline__ void grid_sync(unsigned long long *bar, unsigned long long &target) {
    __syncthreads();
    target += gridDim.x;
    if (threadIdx.x == 0) {
        __threadfence();
        atomicAdd(bar, 1ull);
        while (ld_acquire_u64(bar) < target) {
        }
        __threadfence();
    }
    __syncthreads();
}

__device__ __forceinline__ unsigned long long globaltimer_ns() {
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
}

// View of the per-call lists (raw pointers).
struct ListsView {
    long long *Lt_seg;            // segment id J
    unsigned long long *Lt_mask;  // segment's x bits (nt bits)
    long long *Lt_first;          // first x entry of the segment
    long long *Lt_tbeg;           // first tile of tile column J
    long long *Lt_wpre;           // exclusive tile-work prefix (+ sentinel at nLt)
    long long *Ls_beg;            // first side nonzero of column j
    long long *Ls_wpre;           // exclusive side-work prefix (+ sentinel)
    double *Ls_x;                 // x_j
    int *Ls_col;                  // j
    int *Ct;                      // tile chunk -> first Lt entry
    int *Cs;                      // side chunk -> first Ls entry
    double *xv;                   // x values (double)
    double *xd;                   // x values scattered by column: xd[j] = x_j
};

inline ListsView lists_view(tsmv_ctx *c) {
    ListsView v;
    v.Lt_seg = c->L.Lt_seg.as<long long>();
    v.Lt_mask = c->L.Lt_mask.as<unsigned long long>();
    v.Lt_first = c->L.Lt_first.as<long long>();
    v.Lt_tbeg = c->L.Lt_tbeg.as<long long>();
    v.Lt_wpre = c->L.Lt_wpre.as<long long>();
    v.Ls_beg = c->L.Ls_beg.as<long long>();
    v.Ls_wpre = c->L.Ls_wpre.as<long long>();
    v.Ls_x = c->L.Ls_x.as<double>();
    v.Ls_col = c->L.Ls_col.as<int>();
    v.Ct = c->L.Ct.as<int>();
    v.Cs = c->L.Cs.as<int>();
    v.xv = c->L.xv.as<double>();
    v.xd = c->xdense.as<double>();
    return v;
}

// Write chunk -> entry map for an entry owning work items [w0, w0+w).
template <int LOGC = CHUNK_LOG>
__device__ __forceinline__ void write_chunks(int *C, long long w0, long long w, int entry) {
    constexpr int CH = 1 << LOGC;
    long long c0 = (w0 + CH - 1) >> LOGC;
    long long c1 = (w0 + w + CH - 1) >> LOGC;
    for (long long ch = c0; ch < c1; ++ch) C[ch] = entry;
}

// Warp loads the work-prefix window of a chunk into shared memory:
// win[q] = wpre[s0 + q] for q in [0, CHUNK], +inf past the list end.
// The trip count is warp-uniform on purpose: with a lane-dependent count
// (q = lane; q <= CHUNK) ptxas compiled the following __syncwarp() to a NOP and
// lanes read win[CHUNK] before lane 0 had stored it (found on B200, r1).
template <int LOGC = CHUNK_LOG>
__device__ __forceinline__ void load_window(long long *win, const long long *wpre, long long s0, long long nL,
                                            int lane) {
    constexpr int CH = 1 << LOGC;
#pragma unroll
    for (int q0 = 0; q0 <= CH; q0 += 32) {
        int q = q0 + lane;
        long long idx = s0 + q;
        long long v = idx <= nL ? __ldcg(&wpre[idx]) : 0x7fffffffffffffffLL;
        if (q <= CH) win[q] = v;
    }
    __syncwarp();
}

// Largest q in [0, CHUNK] with win[q] <= i (win[0] <= i guaranteed).
template <int LOGC = CHUNK_LOG>
__device__ __forceinline__ int window_find(const long long *win, long long i) {
    int lo = 0, hi = 1 << LOGC;  // invariant win[lo] <= i, answer in [lo, hi]
    while (lo < hi) {
        int mid = (lo + hi + 1) >> 1;
        if (win[mid] <= i) lo = mid;
        else hi = mid - 1;
    }
    return lo;
}

// Item -> window-entry map of one chunk without a per-item binary search:
// the entries starting strictly inside the chunk are marked in a (1<<LOGC)-bit
// mask (warp OR-reduction, no shared memory); item j of the chunk then belongs
// to window entry popc(mask & bits(0..j)).  Requires every window entry to own
// at least one item (true for the work lists: entries with zero work are not
// listed).  win = the chunk's window (load_window), base = first item.
template <int LOGC>
struct ChunkMap {
    unsigned w[(1 << LOGC) / 32];
    __device__ __forceinline__ void build(const long long *win, long long base, int lane) {
        constexpr int CH = 1 << LOGC, NWD = CH / 32;
        unsigned loc[NWD];
#pragma unroll
        for (int k = 0; k < NWD; ++k) loc[k] = 0u;
#pragma unroll
        for (int v = 0; v < NWD; ++v) {
            const int q = 1 + lane + 32 * v;  // window entries 1..CH
            const long long d = win[q] - base;
            if (d > 0 && d < CH) {
#pragma unroll
                for (int k = 0; k < NWD; ++k)
                    if ((int)(d >> 5) == k) loc[k] |= 1u << (d & 31);
            }
        }
#pragma unroll
        for (int k = 0; k < NWD; ++k) w[k] = __reduce_or_sync(0xffffffffu, loc[k]);
    }
    __device__ __forceinline__ int entry(int j) const {
        constexpr int NWD = (1 << LOGC) / 32;
        int cnt = 0;
        const int wj = j >> 5;
#pragma unroll
        for (int k = 0; k < NWD; ++k) {
            const unsigned m = k < wj ? 0xffffffffu : (k == wj ? ((j & 31) == 31 ? 0xffffffffu : ((2u << (j & 31)) - 1u)) : 0u);
            cnt += __popc(w[k] & m);
        }
        return cnt;
    }
};

// Segment bits of an NT-segment inside uint32 bitmap words.
template <int NT> __device__ __forceinline__ typename Tr<NT>::word_t seg_bits(const uint32_t *bm, long long J) {
    if constexpr (NT == 16) {
        return (uint16_t)(bm[J >> 1] >> ((J & 1) * 16));
    } else if constexpr (NT == 32) {
        return bm[J];
    } else {
        return ((unsigned long long)bm[2 * J + 1] << 32) | bm[2 * J];
    }
}

// OR bits into an NT-segment, returns the previous segment bits.
template <int NT>
__device__ __forceinline__ typename Tr<NT>::word_t seg_or(uint32_t *bm, long long J, typename Tr<NT>::word_t bits) {
    if constexpr (NT == 16) {
        int sh = (J & 1) * 16;
        unsigned old = atomicOr(&bm[J >> 1], (unsigned)bits << sh);
        return (uint16_t)(old >> sh);
    } else if constexpr (NT == 32) {
        return atomicOr(&bm[J], bits);
    } else {
        return atomicOr((unsigned long long *)(bm + 2 * J), bits);
    }
}

template <class W> __device__ __forceinline__ int popc_w(W w) {
    if constexpr (sizeof(W) == 8) return __popcll(w);
    else return __popc((unsigned)w);
}
template <class W> __device__ __forceinline__ int ffs_w(W w) {
    if constexpr (sizeof(W) == 8) return __ffsll((long long)w) - 1;
    else return __ffs((unsigned)w) - 1;
}

template <class W> __device__ __forceinline__ W warp_or(W v) {
    if constexpr (sizeof(W) == 8) {
        unsigned lo = __reduce_or_sync(0xffffffffu, (unsigned)v);
        unsigned hi = __reduce_or_sync(0xffffffffu, (unsigned)(v >> 32));
        return ((W)hi << 32) | lo;
    } else {
        return (W)__reduce_or_sync(0xffffffffu, (unsigned)v);
    }
}


// order-preserving map double -> uint64 (unsigned order == numeric order)
__device__ __forceinline__ unsigned long long ord_key(double x) {
    unsigned long long b = (unsigned long long)__double_as_longlong(x);
    return (b >> 63) ? ~b : (b | 0x8000000000000000ull);
}
__device__ __forceinline__ double ord_val(unsigned long long k) {
    unsigned long long b = (k >> 63) ? (k & 0x7fffffffffffffffull) : ~k;
    return __longlong_as_double((long long)b);
}

}  // namespace tsmv
