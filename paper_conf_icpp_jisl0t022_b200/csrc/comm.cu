// comm.cu -- the NCCL communicator a distributed context owns (SURVEY §8(b)/(e),
// DESIGN.md §8): bootstrap (tsmv_nccl_unique_id), communicator creation inside
// tsmv_create, the replicated global degree arrays the per-level statistics
// need, and the two exchange steps of the row-block partition:
//   * TileBFS: every rank broadcasts the words of its owned segment of the next
//     frontier bitmap, in place, to every other rank (grouped ncclBroadcast = an
//     all-gather-v without padding or a merge copy);
//   * SpMSpV: x is distributed by owner rows; the per-rank counts are
//     all-gathered, then the owned entries are broadcast into one ascending x.
// NCCL is opened with dlopen at first use ("libnccl.so.2": the copy torch has
// already loaded, else the system one; TSMV_NCCL_LIB overrides), so the library
// has no link-time NCCL dependency and single-GPU users never load it.
#include "common.cuh"
#include <dlfcn.h>
#include <nccl.h>
#include <mutex>

namespace tsmv {

namespace {

struct NcclApi {
    void *h = nullptr;
    decltype(&ncclGetUniqueId) getUniqueId = nullptr;
    decltype(&ncclCommInitRank) commInitRank = nullptr;
    decltype(&ncclCommDestroy) commDestroy = nullptr;
    decltype(&ncclAllGather) allGather = nullptr;
    decltype(&ncclAllReduce) allReduce = nullptr;
    decltype(&ncclBroadcast) broadcast = nullptr;
    decltype(&ncclGroupStart) groupStart = nullptr;
    decltype(&ncclGroupEnd) groupEnd = nullptr;
    decltype(&ncclGetErrorString) errStr = nullptr;
    decltype(&ncclGetVersion) getVersion = nullptr;
};

NcclApi g_nccl;
std::mutex g_nccl_mu;

const NcclApi &nccl() {
    std::lock_guard<std::mutex> lk(g_nccl_mu);
    if (g_nccl.h) return g_nccl;
    const char *path = getenv("TSMV_NCCL_LIB");
    void *h = dlopen(path ? path : "libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
    if (!h) {
        set_error("NCCL not available: dlopen(%s): %s", path ? path : "libnccl.so.2", dlerror());
        throw Err{TSMV_ENCCL};
    }
    NcclApi a;
    a.h = h;
#define TSMV_SYM(field, name)                                                 \
    a.field = reinterpret_cast<decltype(a.field)>(dlsym(h, name));            \
    if (!a.field) {                                                           \
        set_error("NCCL symbol %s missing", name);                            \
        throw Err{TSMV_ENCCL};                                                \
    }
    TSMV_SYM(getUniqueId, "ncclGetUniqueId");
    TSMV_SYM(commInitRank, "ncclCommInitRank");
    TSMV_SYM(commDestroy, "ncclCommDestroy");
    TSMV_SYM(allGather, "ncclAllGather");
    TSMV_SYM(allReduce, "ncclAllReduce");
    TSMV_SYM(broadcast, "ncclBroadcast");
    TSMV_SYM(groupStart, "ncclGroupStart");
    TSMV_SYM(groupEnd, "ncclGroupEnd");
    TSMV_SYM(errStr, "ncclGetErrorString");
    TSMV_SYM(getVersion, "ncclGetVersion");
#undef TSMV_SYM
    g_nccl = a;
    return g_nccl;
}

#define TSMV_NCCL(call)                                                                          \
    do {                                                                                         \
        ncclResult_t _r = (call);                                                                \
        if (_r != ncclSuccess) {                                                                 \
            ::tsmv::set_error("%s:%d %s: %s", __FILE__, __LINE__, #call, nccl().errStr(_r));     \
            throw ::tsmv::Err{TSMV_ENCCL};                                                       \
        }                                                                                        \
    } while (0)

__global__ void k_place_rows(const int *__restrict__ src, long long m, long long row_begin, int *__restrict__ dst) {
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < m; i += (long long)gridDim.x * blockDim.x)
        dst[row_begin + i] = src[i];
}
__global__ void k_or_words(uint32_t *__restrict__ V, const uint32_t *__restrict__ F, long long nw) {
    for (long long w = blockIdx.x * (long long)blockDim.x + threadIdx.x; w < nw; w += (long long)gridDim.x * blockDim.x) {
        const uint32_t b = F[w];
        if (b) V[w] |= b;
    }
}
__global__ void k_sum_i32(const int *__restrict__ a, long long n, unsigned long long *__restrict__ out) {
    unsigned long long s = 0;
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x)
        s += (unsigned long long)a[i];
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
    if ((threadIdx.x & 31) == 0 && s) atomicAdd(out, s);
}

int grid_n(long long n) { return (int)std::max<long long>(1, std::min<long long>((n + 255) / 256, 148LL * 16)); }

}  // namespace

bool has_comm(const tsmv_ctx *c) { return c && c->nccl_comm != nullptr; }

// Communicator of a distributed context (collective over the nranks ranks that
// pass the same unique id), then the replicated global degree arrays:
//   outdeg_g[v] = sum over ranks of the local column counts of column v,
//   indeg_g[v]  = row count of global row v (owner's rows placed, summed),
// and nnz_global = sum of indeg_g, so every rank computes |F|, m_f and m_u of a
// level from the (replicated) frontier bitmap alone: no per-level reduction.
void comm_init(tsmv_ctx *c, const void *unique_id, cudaStream_t st) {
    const NcclApi &N = nccl();
    ncclUniqueId id;
    memcpy(&id, unique_id, sizeof(id));
    ncclComm_t comm = nullptr;
    TSMV_NCCL(N.commInitRank(&comm, c->opt.nranks, id, c->opt.rank));
    c->nccl_comm = comm;
    const long long n = c->n;
    c->outdeg_g.alloc(((std::max<int64_t>(n, 1) + 63) / 64 * 64) * 4);
    c->indeg_g.alloc(((std::max<int64_t>(n, 1) + 63) / 64 * 64) * 4);
    TSMV_CUDA(cudaMemsetAsync(c->outdeg_g.p, 0, c->outdeg_g.bytes, st));
    TSMV_CUDA(cudaMemsetAsync(c->indeg_g.p, 0, c->indeg_g.bytes, st));
    k_place_rows<<<grid_n(c->m), 256, 0, st>>>(c->indeg.as<int>(), c->m, c->row_begin, c->indeg_g.as<int>());
    TSMV_CUDA(cudaGetLastError());
    TSMV_NCCL(N.groupStart());
    TSMV_NCCL(N.allReduce(c->outdeg.p, c->outdeg_g.p, (size_t)n, ncclInt32, ncclSum, comm, st));
    TSMV_NCCL(N.allReduce(c->indeg_g.p, c->indeg_g.p, (size_t)n, ncclInt32, ncclSum, comm, st));
    TSMV_NCCL(N.groupEnd());
    DevBuf s;
    s.alloc(8);
    TSMV_CUDA(cudaMemsetAsync(s.p, 0, 8, st));
    k_sum_i32<<<grid_n(n), 256, 0, st>>>(c->indeg_g.as<int>(), n, s.as<unsigned long long>());
    TSMV_CUDA(cudaGetLastError());
    unsigned long long tot = 0;
    TSMV_CUDA(cudaMemcpyAsync(&tot, s.p, 8, cudaMemcpyDeviceToHost, st));
    TSMV_CUDA(cudaStreamSynchronize(st));
    c->nnz_global = (long long)tot;
}

void comm_destroy(tsmv_ctx *c) {
    if (!c->nccl_comm) return;
    try {
        nccl().commDestroy(static_cast<ncclComm_t>(c->nccl_comm));
    } catch (const Err &) {
    }
    c->nccl_comm = nullptr;
}

// Next frontier: every rank's owned words [row_splits[p] / 32, row_splits[p+1] / 32)
// of F are broadcast in place from rank p (splits are multiples of 64 rows), the
// ranks' statistics shares (4 x u64) all-gathered in the same NCCL group, then the
// whole frontier is ORed into the replicated visited bitmap.
void comm_exchange_frontier(tsmv_ctx *c, uint32_t *F, uint32_t *V, long long nwords, const void *stats_send,
                            void *stats_all, cudaStream_t st) {
    const NcclApi &N = nccl();
    ncclComm_t comm = static_cast<ncclComm_t>(c->nccl_comm);
    TSMV_NCCL(N.groupStart());
    for (int p = 0; p < c->opt.nranks; ++p) {
        const long long w0 = c->row_splits[p] >> 5, w1 = (c->row_splits[p + 1] + 31) >> 5;
        if (w1 > w0) TSMV_NCCL(N.broadcast(F + w0, F + w0, (size_t)(w1 - w0), ncclUint32, p, comm, st));
    }
    // every rank's statistics shares of the new frontier ride in the same group
    if (stats_send) TSMV_NCCL(N.allGather(stats_send, stats_all, 4, ncclUint64, comm, st));
    TSMV_NCCL(N.groupEnd());
    k_or_words<<<grid_n(nwords), 256, 0, st>>>(V, F, nwords);
    TSMV_CUDA(cudaGetLastError());
}

// x distributed by owner: all-gather the counts (one 8-byte read on the host),
// then broadcast every rank's entries into one x, ascending because the owners'
// row ranges are.  Returns the global count; *xi / *xv point into ctx buffers.
long long comm_gather_x(tsmv_ctx *c, long long k_local, const int32_t *x_idx, const void *x_val, size_t vb,
                        const int32_t **xi_out, const void **xv_out, cudaStream_t st) {
    const NcclApi &N = nccl();
    ncclComm_t comm = static_cast<ncclComm_t>(c->nccl_comm);
    const int P = c->opt.nranks;
    c->kcounts.ensure((size_t)(P + 1) * 8);
    long long *kc = c->kcounts.as<long long>();
    TSMV_CUDA(cudaMemcpyAsync(kc + P, &k_local, 8, cudaMemcpyHostToDevice, st));
    TSMV_NCCL(N.allGather(kc + P, kc, 1, ncclInt64, comm, st));
    std::vector<long long> cnt(P);
    TSMV_CUDA(cudaMemcpyAsync(cnt.data(), kc, (size_t)P * 8, cudaMemcpyDeviceToHost, st));
    TSMV_CUDA(cudaStreamSynchronize(st));
    long long K = 0;
    for (long long v : cnt) K += v;
    c->xg_idx.ensure((size_t)std::max<long long>(K, 1) * 4);
    c->xg_val.ensure((size_t)std::max<long long>(K, 1) * vb);
    const ncclDataType_t vt = vb == 4 ? ncclFloat32 : ncclFloat64;
    TSMV_NCCL(N.groupStart());
    long long off = 0;
    for (int p = 0; p < P; ++p) {
        if (cnt[p] > 0) {
            const bool me = p == c->opt.rank;
            TSMV_NCCL(N.broadcast(me ? (const void *)x_idx : (const void *)(c->xg_idx.as<int32_t>() + off), c->xg_idx.as<int32_t>() + off, (size_t)cnt[p],
                                  ncclInt32, p, comm, st));
            if (x_val)
                TSMV_NCCL(N.broadcast(me ? x_val : (const void *)(c->xg_val.as<char>() + off * vb), c->xg_val.as<char>() + off * vb, (size_t)cnt[p], vt, p,
                                      comm, st));
        }
        off += cnt[p];
    }
    TSMV_NCCL(N.groupEnd());
    *xi_out = c->xg_idx.as<int32_t>();
    *xv_out = x_val ? c->xg_val.p : nullptr;
    return K;
}

}  // namespace tsmv

extern "C" tsmv_status tsmv_nccl_unique_id(void *out128) {
    using namespace tsmv;
    try {
        TSMV_REQUIRE(out128 != nullptr, "tsmv_nccl_unique_id: NULL out");
        static_assert(sizeof(ncclUniqueId) == 128, "ncclUniqueId is 128 bytes");
        ncclUniqueId id;
        TSMV_NCCL(nccl().getUniqueId(&id));
        memcpy(out128, &id, sizeof(id));
        return TSMV_OK;
    } catch (const Err &e) {
        return e.st;
    }
}
