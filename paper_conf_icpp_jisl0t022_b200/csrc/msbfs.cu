// msbfs.cu -- multi-source TileBFS (the paper's BFS, Alg 3
// P:418-430, run for up to 64 sources at once, the "multiple BFS" workload its
// introduction motivates).
//
// One bit per source in 64-bit vertex words: V[v] (visited by source s), F[v]
// (v is in source s's current frontier), N[v] (found this level).  Every level
// is a bottom-up (Pull-CSC, Alg 7) pass for all sources together:
//   tiles  -- warp per row tile I of the row structure Q; lane = tile t of the
//             group; for every row r of I still missing some source, the row
//             word (plane r) of t names the in-neighbours c, and the
//             frontier words F[16 J_t + c] are ORed (the 16 words of the tile's
//             column segment are one 128-byte line: the tile format turns the
//             bit-parallel pull into coalesced segment reads); column segments
//             without any frontier vertex are skipped by a 1-bit-per-segment map;
//   side   -- thread per vertex over its side in-neighbours, stop once every
//             missing source is found;
//   update -- new = N & ~V: V |= new, next F = new, levels[v][s] = L + 1.
// Levels are those of 64 independent BFS (bit-exact against the oracle's queue
// BFS per source).  nt = 16 contexts (the default) only.
#include "bfs_dev.cuh"
#include <algorithm>
#include <vector>

namespace tsmv {

namespace {

using u64 = unsigned long long;
constexpr int MSB = 256;

__device__ __forceinline__ u64 warp_or64(u64 x) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) x |= __shfl_xor_sync(0xffffffffu, x, o);
    return x;
}

__global__ void k_ms_init(const long long *__restrict__ src, int nsrc, u64 *__restrict__ V, u64 *__restrict__ F,
                          uint32_t *__restrict__ seg, int32_t *__restrict__ levels) {
    const int s = threadIdx.x;
    if (s >= nsrc) return;
    const long long v = src[s];
    atomicOr(&V[v], 1ull << s);
    atomicOr(&F[v], 1ull << s);
    atomicOr(&seg[(v >> 4) >> 5], 1u << ((v >> 4) & 31));
    levels[v * nsrc + s] = 0;
}

// tile part of one bottom-up level (nt = 16), load-balanced over TILES: lane =
// tile t (tiles are sorted by row tile I = tgrp[t]).  For the rows of I that
// still miss some source (rowneed[I]) the row word (plane r) of t names the
// in-neighbours c in column segment J = trow[t]; their frontier words are ORed
// (one 128-byte line per tile).  Lanes holding the same row tile are merged by
// a segmented OR over the warp, and the segment head ORs the result into N.
__global__ void __launch_bounds__(MSB) k_ms_pull_tiles(BfsTiles Q, const u64 *__restrict__ F,
                                                       const uint32_t *__restrict__ seg,
                                                       const uint16_t *__restrict__ rowneed, u64 *__restrict__ N) {
    const int lane = threadIdx.x & 31;
    const long long warp = (blockIdx.x * (long long)blockDim.x + threadIdx.x) >> 5;
    const long long nwarps = ((long long)gridDim.x * blockDim.x) >> 5;
    const uint16_t *planes = (const uint16_t *)Q.planes;
    for (long long tb = warp * 32; tb < Q.T; tb += nwarps * 32) {
        const long long t = tb + lane;
        long long I = -1;
        unsigned rn = 0;
        u64 acc[16];
#pragma unroll
        for (int r = 0; r < 16; ++r) acc[r] = 0ull;
        if (t < Q.T) {
            I = Q.tgrp[t];
            rn = rowneed[I];
            if (rn) {
                const long long J = Q.trow[t];
                if ((seg[J >> 5] >> (J & 31)) & 1u) {
                    const u64 *Fs = F + J * 16;
#pragma unroll
                    for (int r = 0; r < 16; ++r) {
                        if ((rn >> r) & 1u) {
                            unsigned w = planes[(long long)r * Q.T + t];
                            while (w) {
                                const int c = __ffs(w) - 1;
                                w &= w - 1;
                                acc[r] |= __ldg(Fs + c);
                            }
                        }
                    }
                }
            }
        }
        // segmented OR over lanes with the same row tile (contiguous lanes)
        const unsigned same = __match_any_sync(0xffffffffu, I);
        const int last = 31 - __clz(same);
        bool any = false;
#pragma unroll
        for (int r = 0; r < 16; ++r) {
#pragma unroll
            for (int d = 1; d < 32; d <<= 1) {
                const u64 y = __shfl_down_sync(0xffffffffu, acc[r], d);
                if (lane + d <= last) acc[r] |= y;
            }
            any |= acc[r] != 0ull;
        }
        const bool head = I >= 0 && (lane == 0 || ((same >> (lane - 1)) & 1u) == 0u);
        if (head && any) {
#pragma unroll
            for (int r = 0; r < 16; ++r)
                if (acc[r]) atomicOr(&N[I * 16 + r], acc[r]);
        }
    }
}

// side part: in-neighbours u of v in the side CSR of Q.  Vertices with at most
// MS_HEAVY side in-neighbours: thread per vertex, stop once every missing source
// is found; heavier ones (power-law hubs) go to k_ms_pull_side_chunks.
constexpr int MS_HEAVY = 32;  // = the chunk threshold of heavy_side_chunks

template <int NT>
__global__ void __launch_bounds__(MSB) k_ms_pull_side(BfsTiles Q, const u64 *__restrict__ V, const u64 *__restrict__ F,
                                                      u64 *__restrict__ N, long long m, u64 all) {
    for (long long v = blockIdx.x * (long long)blockDim.x + threadIdx.x; v < m; v += (long long)gridDim.x * blockDim.x) {
        if (!((Q.smask[v >> 5] >> (v & 31)) & 1u)) continue;
        const long long p0 = Q.sptr[v], p1 = Q.sptr[v + 1];
        if (p1 - p0 > MS_HEAVY) continue;
        const u64 need = all & ~V[v] & ~N[v];
        if (!need) continue;
        u64 acc = 0ull;
        for (long long p = p0; p < p1; p += 4) {
            int sr[4];
#pragma unroll
            for (int j = 0; j < 4; ++j) sr[j] = p + j < p1 ? Q.srow[p + j] : -1;
#pragma unroll
            for (int j = 0; j < 4; ++j)
                if (p + j < p1) acc |= F[decode_row<NT>(sr[j], Q.hot_list)];
            if ((acc & need) == need) break;
        }
        if (acc & need) N[v] |= acc & need;
    }
}

// heavy side rows in 256-entry chunks (heavy_side_chunks), one warp per chunk,
// merged into N with atomicOr; a chunk stops early once its rows cover every
// source the vertex still misses
template <int NT>
__global__ void __launch_bounds__(MSB) k_ms_pull_side_chunks(BfsTiles Q, const u64 *__restrict__ V,
                                                             const u64 *__restrict__ F, u64 *__restrict__ N,
                                                             const long long *__restrict__ chunks, long long nchunks,
                                                             u64 all) {
    const int lane = threadIdx.x & 31;
    const long long warp = (blockIdx.x * (long long)blockDim.x + threadIdx.x) >> 5;
    const long long nwarps = ((long long)gridDim.x * blockDim.x) >> 5;
    for (long long q = warp; q < nchunks; q += nwarps) {
        const long long e = chunks[q];
        const long long v = e >> 24, i = e & 0xffffff;
        const u64 need = all & ~V[v];
        if (!need) continue;
        const long long p0 = Q.sptr[v] + i * 256, p1 = min(Q.sptr[v + 1], p0 + 256);
        u64 acc = 0ull;
        for (long long pb = p0; pb < p1; pb += 32) {
            if (pb + lane < p1) acc |= F[decode_row<NT>(Q.srow[pb + lane], Q.hot_list)];
            acc = warp_or64(acc);
            if ((acc & need) == need) break;
        }
        if (lane == 0 && (acc & need)) atomicOr(&N[v], acc & need);
    }
}


// new = N & ~V; V |= new; next frontier = new; levels; counts; rowneed[I] =
// rows of row tile I still missing some source (a warp covers 32 consecutive
// vertices = two row tiles)
__global__ void __launch_bounds__(MSB) k_ms_update(u64 *__restrict__ V, u64 *__restrict__ N, u64 *__restrict__ Fn,
                                                   uint32_t *__restrict__ segn, uint16_t *__restrict__ rowneed,
                                                   int32_t *__restrict__ levels, const int *__restrict__ outdeg,
                                                   long long m, int nsrc, int level, u64 all,
                                                   unsigned long long *__restrict__ out) {
    const int lane = threadIdx.x & 31;
    const long long warp = (blockIdx.x * (long long)blockDim.x + threadIdx.x) >> 5;
    const long long nwarps = ((long long)gridDim.x * blockDim.x) >> 5;
    unsigned long long cnt = 0, edges = 0;
    for (long long base = warp * 32; base < m; base += nwarps * 32) {
        const long long v = base + lane;
        bool need = false;
        u64 newbits = 0ull;
        if (v < m) {
            const u64 n = N[v];
            u64 vis = V[v];
            u64 nw = 0ull;
            if (n) {
                nw = n & ~vis;
                N[v] = 0ull;
                if (nw) {
                    vis |= nw;
                    V[v] = vis;
                    atomicOr(&segn[(v >> 4) >> 5], 1u << ((v >> 4) & 31));
                    const int pc = __popcll(nw);
                    cnt += pc;
                    edges += (unsigned long long)pc * (unsigned long long)outdeg[v];
                }
            }
            Fn[v] = nw;
            need = (all & ~vis) != 0ull;
            newbits = nw;
        }
        // levels of the new (vertex, source) pairs: the warp writes one vertex row
        // (nsrc int32) at a time, lane l taking sources l and l + 32
        unsigned todo = __ballot_sync(0xffffffffu, newbits != 0ull);
        while (todo) {
            const int src_lane = __ffs(todo) - 1;
            todo &= todo - 1;
            const u64 nb = __shfl_sync(0xffffffffu, newbits, src_lane);
            const long long row = (base + src_lane) * nsrc;
            if ((nb >> lane) & 1ull) levels[row + lane] = level + 1;
            if (lane + 32 < nsrc && ((nb >> (lane + 32)) & 1ull)) levels[row + lane + 32] = level + 1;
        }
        const unsigned bal = __ballot_sync(0xffffffffu, need);
        if (lane == 0) {
            rowneed[base >> 4] = (uint16_t)(bal & 0xffffu);
            if (base + 16 < m) rowneed[(base >> 4) + 1] = (uint16_t)(bal >> 16);
        }
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        cnt += __shfl_xor_sync(0xffffffffu, cnt, o);
        edges += __shfl_xor_sync(0xffffffffu, edges, o);
    }
    if (lane == 0 && cnt) {
        atomicAdd(&out[0], cnt);
        atomicAdd(&out[1], edges);
    }
}

__global__ void k_ms_src_edges(const long long *__restrict__ src, int nsrc, const int *__restrict__ outdeg,
                               unsigned long long *__restrict__ out) {
    const int s = threadIdx.x;
    if (s < nsrc) atomicAdd(&out[1], (unsigned long long)outdeg[src[s]]);
}

inline int grid_ms(long long n, int maxg) {
    long long g = (n + MSB - 1) / MSB;
    return (int)std::max<long long>(1, std::min<long long>(g, maxg));
}

}  // namespace
}  // namespace tsmv

using namespace tsmv;

extern "C" tsmv_status tsmv_msbfs(tsmv_ctx *c, int32_t nsrc, const int64_t *sources, int32_t *levels,
                                  tsmv_msbfs_stats *stats, void *cuda_stream) {
    try {
        TSMV_REQUIRE(c != nullptr && sources != nullptr && levels != nullptr, "tsmv_msbfs: NULL argument");
        TSMV_REQUIRE(c->bfs_built, "tsmv_msbfs: context built without BFS structures");
        TSMV_REQUIRE(c->opt.nranks == 1, "tsmv_msbfs: single-GPU contexts only");
        TSMV_REQUIRE(nsrc >= 1 && nsrc <= 64, "tsmv_msbfs: nsrc %d out of [1, 64]", (int)nsrc);
        if (c->nt != 16) {
            set_error("tsmv_msbfs: tile_dim 16 contexts only (this one has %d)", c->nt);
            return TSMV_EUNSUPPORTED;
        }
        for (int s = 0; s < nsrc; ++s)
            TSMV_REQUIRE(sources[s] >= 0 && sources[s] < c->n, "tsmv_msbfs: source %lld out of range",
                         (long long)sources[s]);
        TSMV_REQUIRE(is_device_ptr(levels), "tsmv_msbfs: levels must be device memory");
        TSMV_CUDA(cudaSetDevice(c->device));
        cudaStream_t st = (cudaStream_t)cuda_stream;
        const long long m = c->m, nseg = (m + 15) / 16, nsw = (nseg + 31) / 32;
        c->ms_V.ensure(m * 8);
        c->ms_F0.ensure(m * 8);
        c->ms_F1.ensure(m * 8);
        c->ms_N.ensure(m * 8);
        c->ms_seg0.ensure(nsw * 4);
        c->ms_seg1.ensure(nsw * 4);
        c->ms_src.ensure(64 * 8);
        c->ms_out.ensure(2 * 8);
        c->ms_rowneed.ensure(((m + 15) / 16 + 1) * 2);
        heavy_side_chunks(c, st);
        u64 *V = c->ms_V.as<u64>(), *Fa = c->ms_F0.as<u64>(), *Fb = c->ms_F1.as<u64>(), *N = c->ms_N.as<u64>();
        uint32_t *sa = c->ms_seg0.as<uint32_t>(), *sb = c->ms_seg1.as<uint32_t>();
        unsigned long long *out = c->ms_out.as<unsigned long long>();
        const u64 all = nsrc == 64 ? ~0ull : ((1ull << nsrc) - 1ull);
        TSMV_CUDA(cudaEventRecord(c->ev0, st));
        TSMV_CUDA(cudaMemcpyAsync(c->ms_src.p, sources, nsrc * 8, cudaMemcpyHostToDevice, st));
        TSMV_CUDA(cudaMemsetAsync(V, 0, m * 8, st));
        TSMV_CUDA(cudaMemsetAsync(Fa, 0, m * 8, st));
        TSMV_CUDA(cudaMemsetAsync(N, 0, m * 8, st));
        TSMV_CUDA(cudaMemsetAsync(sa, 0, nsw * 4, st));
        TSMV_CUDA(cudaMemsetAsync(levels, 0xff, (size_t)m * nsrc * 4, st));
        TSMV_CUDA(cudaMemsetAsync(c->ms_rowneed.p, 0xff, c->ms_rowneed.bytes, st));  // level 0: every row may need
        TSMV_CUDA(cudaMemsetAsync(out, 0, 16, st));
        k_ms_init<<<1, 64, 0, st>>>(c->ms_src.as<long long>(), nsrc, V, Fa, sa, levels);
        k_ms_src_edges<<<1, 64, 0, st>>>(c->ms_src.as<long long>(), nsrc, c->outdeg.as<int>(), out);
        TSMV_CUDA(cudaGetLastError());
        BfsTiles Q = bfs_tiles(*c->Q);
        const int gmax = c->sm_count * 8;
        long long pairs = nsrc, edges = 0;
        int L = 0;
        std::vector<unsigned long long> h(2);
        while (true) {
            TSMV_CUDA(cudaMemsetAsync(sb, 0, nsw * 4, st));
            uint16_t *rn = c->ms_rowneed.as<uint16_t>();
            if (Q.T) k_ms_pull_tiles<<<grid_ms(Q.T, gmax), MSB, 0, st>>>(Q, Fa, sa, rn, N);
            k_ms_pull_side<16><<<grid_ms(m, gmax), MSB, 0, st>>>(Q, V, Fa, N, m, all);
            if (c->par_nchunks)
                k_ms_pull_side_chunks<16><<<grid_ms(c->par_nchunks * 32, gmax), MSB, 0, st>>>(
                    Q, V, Fa, N, c->par_chunks.as<long long>(), c->par_nchunks, all);
            TSMV_CUDA(cudaMemsetAsync(out, 0, 8, st));  // new pairs of this level (edges keep accumulating)
            k_ms_update<<<grid_ms(m, gmax), MSB, 0, st>>>(V, N, Fb, sb, rn, levels, c->outdeg.as<int>(), m, nsrc, L,
                                                          all, out);
            TSMV_CUDA(cudaGetLastError());
            TSMV_CUDA(cudaMemcpyAsync(h.data(), out, 16, cudaMemcpyDeviceToHost, st));
            TSMV_CUDA(cudaStreamSynchronize(st));
            ++L;
            if (h[0] == 0) break;
            pairs += (long long)h[0];
            std::swap(Fa, Fb);
            std::swap(sa, sb);
        }
        edges = (long long)h[1];
        TSMV_CUDA(cudaEventRecord(c->ev1, st));
        TSMV_CUDA(cudaEventSynchronize(c->ev1));
        if (stats) {
            float ms = 0;
            TSMV_CUDA(cudaEventElapsedTime(&ms, c->ev0, c->ev1));
            stats->nlevels = L;
            stats->pairs_reached = pairs;
            stats->edges_traversed = edges;
            stats->ms = ms;
        }
        return TSMV_OK;
    } catch (const Err &e) {
        return e.st;
    }
}
