// bfs2d.cu -- the per-rank steps of the 2D (processor row x processor column)
// partitioned TileBFS (beyond one GPU's memory; the
// level-synchronous loop is the paper's Alg 3, with the expansion
// y = A x over the OR-AND semiring, as the SpMSpV of the block).
//
// Rank (i, j) of a Pr x Pc grid holds the block A_ij = A[R_i, C_j] as an ordinary
// libtsmv context (local row ids 0..|R_i|, local column ids of the padded column
// space of C_j, DESIGN.md §8 "2D").  A level on rank (i, j) is
//   1. y = A_ij (x) x_j            tsmv_spmspv_async, OR-AND (the flat or the
//                                  row-driven kernel, chosen by x density);
//   2. tsmv_bfs2d_scatter          y's row ids -> a bitmap over R_i;
//   3. caller: all-to-all in processor row i (rank (i, j') receives the words of
//      its sub-piece R_ij' from every rank of the row);
//   4. tsmv_bfs2d_merge            OR the Pc partial bitmaps of R_ij, new = OR &
//                                  ~visited, visited |= new, levels[new] = L + 1,
//                                  new -> this rank's frontier words, |new|;
//   5. caller: all-gather in processor column j of the frontier words of the
//      sub-pieces R_0j .. R_(Pr-1)j = the padded bitmap of C_j;
//   6. tsmv_bfs2d_list             that bitmap -> ascending local column ids = x_j.
// The per-rank state is O(|R_i| / 32 + |C_j| / 32 + |R_ij|) words instead of the
// row-block design's replicated O(n) bitmaps and degree arrays.
#include "common.cuh"

#include <cub/cub.cuh>

namespace tsmv {

namespace {

constexpr int B2D = 256;

__global__ void k_scatter_bits(const int32_t *__restrict__ idx, const int64_t *__restrict__ count, long long cap,
                               uint32_t *__restrict__ words) {
    const long long n = min((long long)*count, cap);
    for (long long e = blockIdx.x * (long long)blockDim.x + threadIdx.x; e < n; e += (long long)gridDim.x * blockDim.x) {
        const int32_t r = idx[e];
        atomicOr(&words[r >> 5], 1u << (r & 31));
    }
}

// warp per 32 consecutive words: lane w computes its word (coalesced), then the
// warp walks the non-zero new words, lane l taking bit l (levels and degree
// loads one line per word)
__global__ void k_merge2d(const uint32_t *__restrict__ segs, int nseg, long long stride, long long nverts,
                          uint32_t *__restrict__ visited, int32_t *__restrict__ levels, int level,
                          uint32_t *__restrict__ front, const int32_t *__restrict__ outdeg,
                          const int32_t *__restrict__ indeg, unsigned long long *__restrict__ stats) {
    const long long nw = (nverts + 31) >> 5;
    const int lane = threadIdx.x & 31;
    const long long nwarps = ((long long)gridDim.x * blockDim.x) >> 5;
    unsigned long long c = 0, so = 0, si = 0;
    for (long long wb = (((long long)blockIdx.x * blockDim.x + threadIdx.x) >> 5) * 32; wb < nw; wb += nwarps * 32) {
        const long long w = wb + lane;
        uint32_t nb = 0;
        if (w < nw) {
            uint32_t acc = 0;
            for (int p = 0; p < nseg; ++p) acc |= segs[p * stride + w];
            const long long v0 = w * 32;
            if (v0 + 32 > nverts) acc &= (1u << (nverts - v0)) - 1u;
            const uint32_t vis = visited[w];
            nb = acc & ~vis;
            front[w] = nb;
            if (nb) visited[w] = vis | nb;
        }
        unsigned nz = __ballot_sync(0xffffffffu, nb != 0u);
        while (nz) {
            const int k = __ffs(nz) - 1;
            nz &= nz - 1;
            const uint32_t b = __shfl_sync(0xffffffffu, nb, k);
            if ((b >> lane) & 1u) {
                const long long v = (wb + k) * 32 + lane;
                levels[v] = level;
                ++c;
                if (outdeg) so += (unsigned long long)outdeg[v];
                if (indeg) si += (unsigned long long)indeg[v];
            }
        }
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        c += __shfl_xor_sync(0xffffffffu, c, o);
        so += __shfl_xor_sync(0xffffffffu, so, o);
        si += __shfl_xor_sync(0xffffffffu, si, o);
    }
    if (lane == 0 && c) {
        atomicAdd(&stats[0], c);
        atomicAdd(&stats[1], so);
        atomicAdd(&stats[2], si);
    }
}

// bitmap -> ascending ids, pass 1: set bits per block of B2D x 4 words
__global__ void __launch_bounds__(B2D) k_list_count(const uint32_t *__restrict__ words, long long nwords,
                                                     long long *__restrict__ bsum) {
    using BR = cub::BlockReduce<long long, B2D>;
    __shared__ typename BR::TempStorage ts;
    const long long w0 = ((long long)blockIdx.x * B2D + threadIdx.x) * 4;
    long long c = 0;
    for (int k = 0; k < 4; ++k)
        if (w0 + k < nwords) c += __popc(words[w0 + k]);
    const long long s = BR(ts).Sum(c);
    if (threadIdx.x == 0) bsum[blockIdx.x] = s;
}

// pass 2 (after an exclusive scan of the block sums): each thread writes the
// ids of its 4 words at its block-exclusive offset; the last block writes the total
__global__ void __launch_bounds__(B2D) k_list_emit(const uint32_t *__restrict__ words, long long nwords,
                                                    const long long *__restrict__ bsum,
                                                    const long long *__restrict__ boff, int32_t *__restrict__ out,
                                                    int64_t *__restrict__ total) {
    using BS = cub::BlockScan<long long, B2D>;
    __shared__ typename BS::TempStorage ts;
    const long long w0 = ((long long)blockIdx.x * B2D + threadIdx.x) * 4;
    uint32_t wv[4];
    long long c = 0;
    for (int k = 0; k < 4; ++k) {
        wv[k] = w0 + k < nwords ? words[w0 + k] : 0u;
        c += __popc(wv[k]);
    }
    long long ex;
    BS(ts).ExclusiveSum(c, ex);
    long long o = boff[blockIdx.x] + ex;
    for (int k = 0; k < 4; ++k) {
        uint32_t b = wv[k];
        while (b) {
            const int r = __ffs(b) - 1;
            b &= b - 1;
            out[o++] = (int32_t)((w0 + k) * 32 + r);
        }
    }
    if (blockIdx.x == gridDim.x - 1 && threadIdx.x == 0) *total = boff[blockIdx.x] + bsum[blockIdx.x];
}

inline int grid2d(long long n, int maxg) {
    long long g = (n + B2D - 1) / B2D;
    return (int)std::max<long long>(1, std::min<long long>(g, maxg));
}

}  // namespace

}  // namespace tsmv

using namespace tsmv;

extern "C" tsmv_status tsmv_bfs2d_scatter(tsmv_ctx *c, const int32_t *y_idx, const int64_t *y_nnz, int64_t y_cap,
                                          uint32_t *words, int64_t nwords, void *cuda_stream) {
    try {
        TSMV_REQUIRE(c && y_idx && y_nnz && words, "tsmv_bfs2d_scatter: NULL argument");
        TSMV_REQUIRE(y_cap >= 0 && nwords >= (c->m + 31) / 32,
                     "tsmv_bfs2d_scatter: nwords %lld < ceil(rows / 32) = %lld", (long long)nwords,
                     (long long)((c->m + 31) / 32));
        TSMV_REQUIRE(is_device_ptr(y_idx) && is_device_ptr(y_nnz) && is_device_ptr(words),
                     "tsmv_bfs2d_scatter: device memory expected");
        TSMV_CUDA(cudaSetDevice(c->device));
        cudaStream_t st = (cudaStream_t)cuda_stream;
        TSMV_CUDA(cudaMemsetAsync(words, 0, (size_t)nwords * 4, st));
        k_scatter_bits<<<grid2d(std::max<int64_t>(y_cap, 1), c->sm_count * 8), B2D, 0, st>>>(y_idx, y_nnz, y_cap,
                                                                                             words);
        TSMV_CUDA(cudaGetLastError());
        return TSMV_OK;
    } catch (const Err &e) {
        return e.st;
    }
}

extern "C" tsmv_status tsmv_bfs2d_merge(tsmv_ctx *c, const uint32_t *segs, int32_t nseg, int64_t stride_words,
                                        int64_t nverts, uint32_t *visited, int32_t *levels, int32_t level,
                                        uint32_t *front_out, const int32_t *outdeg, const int32_t *indeg,
                                        int64_t *stats_dev, void *cuda_stream) {
    try {
        TSMV_REQUIRE(c && segs && visited && levels && front_out && stats_dev, "tsmv_bfs2d_merge: NULL argument");
        TSMV_REQUIRE(nseg >= 1 && nverts >= 0 && stride_words >= (nverts + 31) / 32,
                     "tsmv_bfs2d_merge: nseg %d, stride_words %lld < ceil(nverts / 32)", nseg,
                     (long long)stride_words);
        TSMV_REQUIRE(is_device_ptr(segs) && is_device_ptr(visited) && is_device_ptr(levels) &&
                         is_device_ptr(front_out) && is_device_ptr(stats_dev) &&
                         (!outdeg || is_device_ptr(outdeg)) && (!indeg || is_device_ptr(indeg)),
                     "tsmv_bfs2d_merge: device memory expected");
        TSMV_CUDA(cudaSetDevice(c->device));
        cudaStream_t st = (cudaStream_t)cuda_stream;
        TSMV_CUDA(cudaMemsetAsync(stats_dev, 0, 3 * 8, st));
        if (nverts > 0)
            k_merge2d<<<grid2d((nverts + 31) / 32, c->sm_count * 8), B2D, 0, st>>>(
                segs, nseg, stride_words, nverts, visited, levels, level, front_out, outdeg, indeg,
                reinterpret_cast<unsigned long long *>(stats_dev));
        TSMV_CUDA(cudaGetLastError());
        return TSMV_OK;
    } catch (const Err &e) {
        return e.st;
    }
}

extern "C" tsmv_status tsmv_bfs2d_list(tsmv_ctx *c, const uint32_t *words, int64_t nbits, int32_t *idx_out,
                                       int64_t *count_out, void *cuda_stream) {
    try {
        TSMV_REQUIRE(c && words && idx_out && count_out, "tsmv_bfs2d_list: NULL argument");
        TSMV_REQUIRE(nbits >= 0 && nbits <= (int64_t)INT32_MAX + 1, "tsmv_bfs2d_list: nbits out of range");
        TSMV_REQUIRE(is_device_ptr(words) && is_device_ptr(idx_out), "tsmv_bfs2d_list: device memory expected");
        TSMV_CUDA(cudaSetDevice(c->device));
        cudaStream_t st = (cudaStream_t)cuda_stream;
        const long long nwords = (nbits + 31) / 32;
        const long long nb = std::max<long long>(1, (nwords + 4LL * B2D - 1) / (4LL * B2D));
        c->b2d_bsum.ensure(nb * 8);
        c->b2d_boff.ensure(nb * 8);
        c->b2d_total.ensure(8);
        size_t tb = 0;
        TSMV_CUDA(cub::DeviceScan::ExclusiveSum(nullptr, tb, c->b2d_bsum.as<long long>(), c->b2d_boff.as<long long>(),
                                                (int)nb, st));
        c->b2d_temp.ensure(tb);
        k_list_count<<<(unsigned)nb, B2D, 0, st>>>(words, nwords, c->b2d_bsum.as<long long>());
        TSMV_CUDA(cudaGetLastError());
        TSMV_CUDA(cub::DeviceScan::ExclusiveSum(c->b2d_temp.p, tb, c->b2d_bsum.as<long long>(),
                                                c->b2d_boff.as<long long>(), (int)nb, st));
        k_list_emit<<<(unsigned)nb, B2D, 0, st>>>(words, nwords, c->b2d_bsum.as<long long>(),
                                                  c->b2d_boff.as<long long>(), idx_out, c->b2d_total.as<int64_t>());
        TSMV_CUDA(cudaGetLastError());
        if (is_device_ptr(count_out)) {
            TSMV_CUDA(cudaMemcpyAsync(count_out, c->b2d_total.p, 8, cudaMemcpyDeviceToDevice, st));
        } else {
            TSMV_CUDA(cudaMemcpyAsync(count_out, c->b2d_total.p, 8, cudaMemcpyDeviceToHost, st));
            TSMV_CUDA(cudaStreamSynchronize(st));
        }
        return TSMV_OK;
    } catch (const Err &e) {
        return e.st;
    }
}
