// builder.cu -- CSR -> tiled format (Sec 3.2.1
// P:481-513, Sec 3.2.3; conversion cost Sec 4.6).
//
// Device pipeline (all on the caller's stream):
//   1. per-nonzero tile key  ((J*nTR + I) << 2*LOG) | (c << LOG) | r
//      (tile column major, then tile row, then column-major inside the tile);
//   2. CUB radix sort of (key, value);
//   3. tile heads -> tile ids (scan) -> tile starts / nnz per tile;
//   4. classify: nnz <= sparse_tile_max_nnz -> side matrix (R12);
//   5. one thread per tile writes the tile descriptors (row, col, nnz offset,
//      column mask), the packed in-tile indices + values and the BFS bit planes
//      (nt words of nt bits per tile);
//   6. side entries re-sorted by (column, row) -> side CSC.
#include "common.cuh"
#include <cub/cub.cuh>
#include <algorithm>
#include <vector>

namespace tsmv {

namespace {

struct CubTemp {
    DevBuf buf;
    void *get(size_t b) {
        buf.ensure(b);
        return buf.p;
    }
};

template <int NT>
__global__ void k_keys(const int32_t *__restrict__ rows, const int32_t *__restrict__ cols, int64_t nnz,
                       int64_t nTR, unsigned long long *__restrict__ keys) {
    constexpr int LOG = Tr<NT>::LOG;
    for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < nnz;
         e += (int64_t)gridDim.x * blockDim.x) {
        unsigned long long r = (unsigned)rows[e], c = (unsigned)cols[e];
        unsigned long long tile = (c >> LOG) * (unsigned long long)nTR + (r >> LOG);
        keys[e] = (tile << (2 * LOG)) | ((c & (NT - 1)) << LOG) | (r & (NT - 1));
    }
}

template <int NT>
__global__ void k_heads(const unsigned long long *__restrict__ keys, int64_t nnz, int32_t *__restrict__ head) {
    constexpr int LOG = Tr<NT>::LOG;
    for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < nnz;
         e += (int64_t)gridDim.x * blockDim.x)
        head[e] = (e == 0 || (keys[e] >> (2 * LOG)) != (keys[e - 1] >> (2 * LOG))) ? 1 : 0;
}

__global__ void k_starts(const int32_t *__restrict__ head, const int32_t *__restrict__ tid, int64_t nnz,
                         int64_t Tall, int64_t *__restrict__ starts) {
    for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < nnz;
         e += (int64_t)gridDim.x * blockDim.x) {
        if (head[e]) starts[tid[e] - 1] = e;
        if (e == 0) starts[Tall] = nnz;
    }
}

__global__ void k_classify(const int64_t *__restrict__ starts, int64_t Tall, int thr,
                           int32_t *__restrict__ dflag, int64_t *__restrict__ dnz, int64_t *__restrict__ snz) {
    for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < Tall;
         t += (int64_t)gridDim.x * blockDim.x) {
        int64_t cnt = starts[t + 1] - starts[t];
        bool dense = cnt > thr;
        dflag[t] = dense;
        dnz[t] = dense ? cnt : 0;
        snz[t] = dense ? 0 : cnt;
    }
}

template <int NT, class V>
__global__ void k_fill_tiles(const unsigned long long *__restrict__ keys, const V *__restrict__ vals,
                             const int64_t *__restrict__ starts, int64_t Tall, int64_t nTR, int64_t T,
                             const int32_t *__restrict__ dord, const int64_t *__restrict__ dpos,
                             const int64_t *__restrict__ spos, int64_t dimR,
                             int32_t *__restrict__ trow, int32_t *__restrict__ tgrp,
                             typename Tr<NT>::word_t *__restrict__ mask, int64_t *__restrict__ off,
                             typename Tr<NT>::idx_t *__restrict__ idx, V *__restrict__ dval,
                             typename Tr<NT>::word_t *__restrict__ planes,
                             unsigned long long *__restrict__ skey, V *__restrict__ sval,
                             int32_t *__restrict__ colcnt, TileDesc *__restrict__ desc,
                             typename Tr<NT>::cs_t *__restrict__ cstart, const int32_t *__restrict__ hot_map) {
    using word_t = typename Tr<NT>::word_t;
    using idx_t = typename Tr<NT>::idx_t;
    constexpr int LOG = Tr<NT>::LOG;
    for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < Tall;
         t += (int64_t)gridDim.x * blockDim.x) {
        int64_t s0 = starts[t], s1 = starts[t + 1];
        unsigned long long tile = keys[s0] >> (2 * LOG);
        int64_t J = (int64_t)(tile / (unsigned long long)nTR), I = (int64_t)(tile % (unsigned long long)nTR);
        bool dense = (t + 1 < Tall ? dord[t + 1] : T) != dord[t];
        if (dense) {
            int64_t d = dord[t];
            int64_t p0 = dpos[t];
            word_t mk = 0;
            int next_c = 0;  // columns < next_c have their start written
            for (int64_t e = s0; e < s1; ++e) {
                unsigned c = (unsigned)((keys[e] >> LOG) & (NT - 1));
                unsigned r = (unsigned)(keys[e] & (NT - 1));
                for (; next_c <= (int)c; ++next_c) cstart[d * NT + next_c] = (typename Tr<NT>::cs_t)(e - s0);
                mk |= (word_t)1 << c;
                idx[p0 + (e - s0)] = (idx_t)((c << LOG) | r);
                if (dval) dval[p0 + (e - s0)] = vals[e];
                if (planes) planes[(int64_t)c * T + d] |= (word_t)1 << r;
            }
            for (; next_c < NT; ++next_c) cstart[d * NT + next_c] = (typename Tr<NT>::cs_t)(s1 - s0);
            trow[d] = (int32_t)I;
            tgrp[d] = (int32_t)J;
            mask[d] = mk;
            off[d] = p0;
            TileDesc td;
            td.off = p0;
            td.trow = (hot_map && hot_map[I] >= 0) ? ~hot_map[I] : (int)I;
            td.nnz = (int)(s1 - s0);
            desc[d] = td;
            atomicAdd(&colcnt[J], 1);
        } else {
            int64_t q0 = spos[t];
            for (int64_t e = s0; e < s1; ++e) {
                unsigned long long c = (keys[e] >> LOG) & (NT - 1);
                unsigned long long r = keys[e] & (NT - 1);
                unsigned long long gc = (unsigned long long)J * NT + c, gr = (unsigned long long)I * NT + r;
                skey[q0 + (e - s0)] = gc * (unsigned long long)dimR + gr;
                if (sval) sval[q0 + (e - s0)] = vals[e];
            }
        }
    }
}

__global__ void k_side_split(const unsigned long long *__restrict__ skey, int64_t S, int64_t dimR,
                             int32_t *__restrict__ srow, int32_t *__restrict__ scnt,
                             const int32_t *__restrict__ hot_map, int nt) {
    for (int64_t q = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; q < S;
         q += (int64_t)gridDim.x * blockDim.x) {
        unsigned long long k = skey[q];
        int32_t row = (int32_t)(k % (unsigned long long)dimR);
        if (hot_map) {
            int32_t h = hot_map[row / nt];
            if (h >= 0) row = ~(h * nt + row % nt);
        }
        srow[q] = row;
        atomicAdd(&scnt[k / (unsigned long long)dimR], 1);
    }
}

__global__ void k_widen_scan_input(const int32_t *__restrict__ in, int64_t n, int64_t *__restrict__ out) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        out[i] = in[i];
}

inline int grid_for(int64_t n, int bs = 256) {
    int64_t g = (n + bs - 1) / bs;
    if (g < 1) g = 1;
    if (g > 148 * 32) g = 148 * 32;
    return (int)g;
}

template <class T> T read1(const T *dptr, cudaStream_t st) {
    T h{};
    TSMV_CUDA(cudaMemcpyAsync(&h, dptr, sizeof(T), cudaMemcpyDeviceToHost, st));
    TSMV_CUDA(cudaStreamSynchronize(st));
    return h;
}

// smask word w: bit r set iff side column 32w + r is non-empty
__global__ void k_side_occupancy(const int64_t *__restrict__ sptr, int64_t dimC, uint32_t *__restrict__ smask) {
    for (int64_t w = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; w < (dimC + 31) / 32;
         w += (int64_t)gridDim.x * blockDim.x) {
        uint32_t m = 0;
        for (int r = 0; r < 32 && w * 32 + r < dimC; ++r)
            if (sptr[w * 32 + r + 1] > sptr[w * 32 + r]) m |= 1u << r;
        smask[w] = m;
    }
}

// pmask[J] |= bit c for every plane c that is non-empty in a tile of group J
template <int NT>
__global__ void k_plane_occupancy(const typename Tr<NT>::word_t *__restrict__ planes, const int32_t *__restrict__ tgrp,
                                  int64_t T, unsigned long long *__restrict__ pmask) {
    for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < T; t += (int64_t)gridDim.x * blockDim.x) {
        unsigned long long m = 0;
#pragma unroll 4
        for (int c = 0; c < NT; ++c)
            if (planes[(int64_t)c * T + t]) m |= 1ull << c;
        atomicOr(&pmask[tgrp[t]], m);
    }
}

// counts (int32[n]) -> ptr (int64[n+1]) exclusive prefix
void counts_to_ptr(const int32_t *cnt, int64_t n, int64_t *ptr, CubTemp &tmp, cudaStream_t st) {
    DevBuf wide;
    wide.alloc((n + 1) * sizeof(int64_t));
    TSMV_CUDA(cudaMemsetAsync(wide.p, 0, (n + 1) * sizeof(int64_t), st));
    if (n > 0) k_widen_scan_input<<<grid_for(n), 256, 0, st>>>(cnt, n, wide.as<int64_t>());
    size_t tb = 0;
    cub::DeviceScan::ExclusiveSum(nullptr, tb, wide.as<int64_t>(), ptr, n + 1, st);
    cub::DeviceScan::ExclusiveSum(tmp.get(tb), tb, wide.as<int64_t>(), ptr, n + 1, st);
    TSMV_CUDA(cudaGetLastError());
    TSMV_CUDA(cudaStreamSynchronize(st));
}

template <int NT, class V>
void build_nt(TileSet &S, const int32_t *rows, const int32_t *cols, const V *vals, int64_t nnz, int64_t dimR,
              int64_t dimC, int thr, bool want_planes, cudaStream_t st, const int32_t *hot_map) {
    using word_t = typename Tr<NT>::word_t;
    using idx_t = typename Tr<NT>::idx_t;
    constexpr int LOG = Tr<NT>::LOG;
    CubTemp tmp;
    S.dimR = dimR;
    S.dimC = dimC;
    S.nTR = (dimR + NT - 1) / NT;
    S.nTC = (dimC + NT - 1) / NT;
    S.has_vals = vals != nullptr;
    S.has_planes = want_planes;

    // 1-2. keys + sort
    DevBuf kin, kout, vin, vout;
    kin.alloc(nnz * 8);
    kout.alloc(nnz * 8);
    if (nnz) k_keys<NT><<<grid_for(nnz), 256, 0, st>>>(rows, cols, nnz, S.nTR, kin.as<unsigned long long>());
    unsigned long long maxtile = (unsigned long long)S.nTC * (unsigned long long)S.nTR;
    int end_bit = 2 * LOG;
    while ((1ull << (end_bit - 2 * LOG)) < maxtile && end_bit < 64) ++end_bit;
    size_t tb = 0;
    if (vals) {
        vin.alloc(nnz * sizeof(V));
        vout.alloc(nnz * sizeof(V));
        TSMV_CUDA(cudaMemcpyAsync(vin.p, vals, nnz * sizeof(V), cudaMemcpyDeviceToDevice, st));
        cub::DeviceRadixSort::SortPairs(nullptr, tb, kin.as<unsigned long long>(), kout.as<unsigned long long>(),
                                        vin.as<V>(), vout.as<V>(), nnz, 0, end_bit, st);
        cub::DeviceRadixSort::SortPairs(tmp.get(tb), tb, kin.as<unsigned long long>(),
                                        kout.as<unsigned long long>(), vin.as<V>(), vout.as<V>(), nnz, 0,
                                        end_bit, st);
        vin.release();
    } else {
        cub::DeviceRadixSort::SortKeys(nullptr, tb, kin.as<unsigned long long>(), kout.as<unsigned long long>(),
                                       nnz, 0, end_bit, st);
        cub::DeviceRadixSort::SortKeys(tmp.get(tb), tb, kin.as<unsigned long long>(),
                                       kout.as<unsigned long long>(), nnz, 0, end_bit, st);
    }
    TSMV_CUDA(cudaGetLastError());
    kin.release();
    const unsigned long long *keys = kout.as<unsigned long long>();

    // 3. tiles
    DevBuf head, tid, starts;
    head.alloc(nnz * 4);
    tid.alloc(nnz * 4);
    int64_t Tall = 0;
    if (nnz) {
        k_heads<NT><<<grid_for(nnz), 256, 0, st>>>(keys, nnz, head.as<int32_t>());
        cub::DeviceScan::InclusiveSum(nullptr, tb, head.as<int32_t>(), tid.as<int32_t>(), nnz, st);
        cub::DeviceScan::InclusiveSum(tmp.get(tb), tb, head.as<int32_t>(), tid.as<int32_t>(), nnz, st);
        TSMV_CUDA(cudaGetLastError());
        Tall = read1(tid.as<int32_t>() + nnz - 1, st);
    }
    S.n_tiles_all = Tall;
    starts.alloc((Tall + 1) * 8);
    if (nnz) k_starts<<<grid_for(nnz), 256, 0, st>>>(head.as<int32_t>(), tid.as<int32_t>(), nnz, Tall,
                                                      starts.as<int64_t>());
    else TSMV_CUDA(cudaMemsetAsync(starts.p, 0, 8, st));
    head.release();
    tid.release();

    // 4. classify
    DevBuf dflag, dnz, snz, dord, dpos, spos;
    dflag.alloc((Tall + 1) * 4);
    dnz.alloc((Tall + 1) * 8);
    snz.alloc((Tall + 1) * 8);
    dord.alloc((Tall + 1) * 4);
    dpos.alloc((Tall + 1) * 8);
    spos.alloc((Tall + 1) * 8);
    TSMV_CUDA(cudaMemsetAsync(dflag.p, 0, (Tall + 1) * 4, st));
    TSMV_CUDA(cudaMemsetAsync(dnz.p, 0, (Tall + 1) * 8, st));
    TSMV_CUDA(cudaMemsetAsync(snz.p, 0, (Tall + 1) * 8, st));
    if (Tall) k_classify<<<grid_for(Tall), 256, 0, st>>>(starts.as<int64_t>(), Tall, thr, dflag.as<int32_t>(),
                                                          dnz.as<int64_t>(), snz.as<int64_t>());
    cub::DeviceScan::ExclusiveSum(nullptr, tb, dflag.as<int32_t>(), dord.as<int32_t>(), Tall + 1, st);
    cub::DeviceScan::ExclusiveSum(tmp.get(tb), tb, dflag.as<int32_t>(), dord.as<int32_t>(), Tall + 1, st);
    cub::DeviceScan::ExclusiveSum(nullptr, tb, dnz.as<int64_t>(), dpos.as<int64_t>(), Tall + 1, st);
    cub::DeviceScan::ExclusiveSum(tmp.get(tb), tb, dnz.as<int64_t>(), dpos.as<int64_t>(), Tall + 1, st);
    cub::DeviceScan::ExclusiveSum(nullptr, tb, snz.as<int64_t>(), spos.as<int64_t>(), Tall + 1, st);
    cub::DeviceScan::ExclusiveSum(tmp.get(tb), tb, snz.as<int64_t>(), spos.as<int64_t>(), Tall + 1, st);
    TSMV_CUDA(cudaGetLastError());
    int64_t T = read1(dord.as<int32_t>() + Tall, st);
    int64_t DN = read1(dpos.as<int64_t>() + Tall, st);
    int64_t SN = read1(spos.as<int64_t>() + Tall, st);
    S.T = T;
    S.dense_nnz = DN;
    S.side_nnz = SN;
    dflag.release();
    dnz.release();
    snz.release();

    // 5. fill
    S.trow.alloc(T * 4);
    S.tgrp.alloc(T * 4);
    S.mask.alloc(T * sizeof(word_t));
    S.off.alloc((T + 1) * 8);
    S.idx.alloc(DN * sizeof(idx_t));
    S.desc.alloc(T * sizeof(TileDesc));
    S.cstart.alloc((size_t)T * NT * sizeof(typename Tr<NT>::cs_t));
    if (vals) S.val.alloc(DN * sizeof(V));
    if (want_planes) {
        S.planes.alloc((size_t)NT * T * sizeof(word_t));
        TSMV_CUDA(cudaMemsetAsync(S.planes.p, 0, (size_t)NT * T * sizeof(word_t), st));
    }
    DevBuf skey, sval_tmp, colcnt;
    skey.alloc(SN * 8);
    if (vals) sval_tmp.alloc(SN * sizeof(V));
    colcnt.alloc((S.nTC + 1) * 4);
    TSMV_CUDA(cudaMemsetAsync(colcnt.p, 0, (S.nTC + 1) * 4, st));
    if (Tall)
        k_fill_tiles<NT, V><<<grid_for(Tall, 128), 128, 0, st>>>(
            keys, vals ? vout.as<V>() : nullptr, starts.as<int64_t>(), Tall, S.nTR, T, dord.as<int32_t>(),
            dpos.as<int64_t>(), spos.as<int64_t>(), dimR, S.trow.as<int32_t>(), S.tgrp.as<int32_t>(),
            S.mask.as<word_t>(), S.off.as<int64_t>(), S.idx.as<idx_t>(), vals ? S.val.as<V>() : nullptr,
            want_planes ? S.planes.as<word_t>() : nullptr, skey.as<unsigned long long>(),
            vals ? sval_tmp.as<V>() : nullptr, colcnt.as<int32_t>(), S.desc.as<TileDesc>(),
            S.cstart.as<typename Tr<NT>::cs_t>(), hot_map);
    TSMV_CUDA(cudaGetLastError());
    TSMV_CUDA(cudaMemcpyAsync(S.off.as<int64_t>() + T, &DN, 8, cudaMemcpyHostToDevice, st));
    S.ptr.alloc((S.nTC + 1) * 8);
    counts_to_ptr(colcnt.as<int32_t>(), S.nTC, S.ptr.as<int64_t>(), tmp, st);
    if (want_planes) {
        S.pmask.alloc(std::max<int64_t>(S.nTC, 1) * 8);
        TSMV_CUDA(cudaMemsetAsync(S.pmask.p, 0, S.pmask.bytes, st));
        if (T)
            k_plane_occupancy<NT><<<grid_for(T), 256, 0, st>>>(S.planes.as<word_t>(), S.tgrp.as<int32_t>(), T,
                                                               S.pmask.as<unsigned long long>());
        TSMV_CUDA(cudaGetLastError());
    }
    kout.release();
    vout.release();
    starts.release();
    dord.release();
    dpos.release();
    spos.release();
    colcnt.release();

    // 6. side CSC
    DevBuf skey2, sval2, scnt;
    skey2.alloc(SN * 8);
    if (vals) sval2.alloc(SN * sizeof(V));
    if (SN) {
        if (vals) {
            cub::DeviceRadixSort::SortPairs(nullptr, tb, skey.as<unsigned long long>(),
                                            skey2.as<unsigned long long>(), sval_tmp.as<V>(), sval2.as<V>(), SN,
                                            0, 64, st);
            cub::DeviceRadixSort::SortPairs(tmp.get(tb), tb, skey.as<unsigned long long>(),
                                            skey2.as<unsigned long long>(), sval_tmp.as<V>(), sval2.as<V>(), SN,
                                            0, 64, st);
        } else {
            cub::DeviceRadixSort::SortKeys(nullptr, tb, skey.as<unsigned long long>(),
                                           skey2.as<unsigned long long>(), SN, 0, 64, st);
            cub::DeviceRadixSort::SortKeys(tmp.get(tb), tb, skey.as<unsigned long long>(),
                                           skey2.as<unsigned long long>(), SN, 0, 64, st);
        }
        TSMV_CUDA(cudaGetLastError());
    }
    skey.release();
    sval_tmp.release();
    S.srow.alloc(SN * 4);
    scnt.alloc((dimC + 1) * 4);
    TSMV_CUDA(cudaMemsetAsync(scnt.p, 0, (dimC + 1) * 4, st));
    if (SN) k_side_split<<<grid_for(SN), 256, 0, st>>>(skey2.as<unsigned long long>(), SN, dimR,
                                                        S.srow.as<int32_t>(), scnt.as<int32_t>(), hot_map, NT);
    TSMV_CUDA(cudaGetLastError());
    S.sptr.alloc(((dimC + 63) / 64 * 64 + 1) * 8);  // padded: whole-segment vector loads (k_fscan)
    counts_to_ptr(scnt.as<int32_t>(), dimC, S.sptr.as<int64_t>(), tmp, st);
    if (want_planes) {
        const int64_t nw = (dimC + 31) / 32;
        S.smask.alloc(std::max<int64_t>(nw, 1) * 4);
        if (nw) k_side_occupancy<<<grid_for(nw), 256, 0, st>>>(S.sptr.as<int64_t>(), dimC, S.smask.as<uint32_t>());
        TSMV_CUDA(cudaGetLastError());
    }
    if (vals) S.sval.p = sval2.p, S.sval.bytes = sval2.bytes, sval2.p = nullptr, sval2.bytes = 0;
    TSMV_CUDA(cudaStreamSynchronize(st));
}

__global__ void k_keys_pattern(const int32_t *__restrict__ rows, const int32_t *__restrict__ cols, int64_t nnz,
                               int64_t n, bool transpose, unsigned long long *__restrict__ keys) {
    for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < nnz;
         e += (int64_t)gridDim.x * blockDim.x) {
        unsigned long long r = (unsigned)rows[e], c = (unsigned)cols[e];
        keys[e] = transpose ? c * (unsigned long long)n + r : r * (unsigned long long)n + c;
    }
}

__global__ void k_cmp(const unsigned long long *__restrict__ a, const unsigned long long *__restrict__ b,
                      int64_t nnz, int *__restrict__ diff) {
    for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < nnz;
         e += (int64_t)gridDim.x * blockDim.x)
        if (a[e] != b[e]) *diff = 1;
}

// row_ptr checks (thread per row), in-degrees, and the row id of every non-empty
// row's first nonzero (the max-scan of these heads gives the row of every nonzero)
__global__ void k_check_rows(const int64_t *__restrict__ row_ptr, int64_t m, int64_t nnz, int *__restrict__ bad,
                             int32_t *__restrict__ indeg, int32_t *__restrict__ heads) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < m; i += (int64_t)gridDim.x * blockDim.x) {
        const int64_t p0 = row_ptr[i], p1 = row_ptr[i + 1];
        if (p0 > p1 || p0 < 0 || p1 > nnz || (i == 0 && p0 != 0) || (i == m - 1 && p1 != nnz)) {
            *bad = 1;
            continue;
        }
        indeg[i] = (int32_t)(p1 - p0);
        if (p1 > p0) heads[p0] = (int32_t)i;
    }
}
// columns strictly ascending inside a row and < ncols (thread per nonzero)
__global__ void k_check_cols(const int32_t *__restrict__ rows, const int32_t *__restrict__ col, int64_t nnz,
                             int64_t ncols, int *__restrict__ bad) {
    for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < nnz; e += (int64_t)gridDim.x * blockDim.x) {
        const int32_t cc = col[e];
        if (cc < 0 || cc >= ncols || (e > 0 && rows[e] == rows[e - 1] && cc <= col[e - 1])) *bad = 2;
    }
}
struct MaxI32 {
    __device__ __forceinline__ int32_t operator()(int32_t a, int32_t b) const { return a > b ? a : b; }
};

__global__ void k_colcount(const int32_t *__restrict__ col, int64_t nnz, int32_t *__restrict__ cnt) {
    for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < nnz; e += (int64_t)gridDim.x * blockDim.x)
        atomicAdd(&cnt[col[e]], 1);
}

}  // namespace

// Validate the CSR (row_ptr monotone, columns strictly ascending in range),
// expand row ids per nonzero, in-degree (row counts) and out-degree (column counts).
void prepare_csr(tsmv_ctx *c, const int64_t *row_ptr, const int32_t *col_idx, int32_t *rows, cudaStream_t st) {
    DevBuf bad;
    bad.alloc(4);
    TSMV_CUDA(cudaMemsetAsync(bad.p, 0, 4, st));
    c->indeg.alloc(std::max<int64_t>(c->m, 1) * 4);
    c->outdeg.alloc(((std::max<int64_t>(c->n, 1) + 63) / 64 * 64) * 4);  // padded for segment vector loads
    TSMV_CUDA(cudaMemsetAsync(c->indeg.p, 0, c->indeg.bytes, st));
    TSMV_CUDA(cudaMemsetAsync(c->outdeg.p, 0, c->outdeg.bytes, st));
    // row checks + row heads (thread per row), row of every nonzero by a max-scan
    // of the heads, column checks (thread per nonzero): O(nnz) with no per-row
    // serial loop (a power-law row used to serialise one thread for milliseconds)
    DevBuf heads;
    if (c->nnz) {
        heads.alloc(c->nnz * 4);
        TSMV_CUDA(cudaMemsetAsync(heads.p, 0, c->nnz * 4, st));
    }
    if (c->m) k_check_rows<<<grid_for(c->m), 256, 0, st>>>(row_ptr, c->m, c->nnz, bad.as<int>(),
                                                          c->indeg.as<int32_t>(), c->nnz ? heads.as<int32_t>() : nullptr);
    TSMV_CUDA(cudaGetLastError());
    int b = read1(bad.as<int>(), st);
    TSMV_REQUIRE(b == 0, "tsmv_create: row_ptr not monotone / inconsistent with nnz");
    if (c->nnz) {
        size_t tb = 0;
        TSMV_CUDA(cub::DeviceScan::InclusiveScan(nullptr, tb, heads.as<int32_t>(), rows, MaxI32(), c->nnz, st));
        DevBuf tmp;
        tmp.alloc(tb);
        TSMV_CUDA(cub::DeviceScan::InclusiveScan(tmp.p, tb, heads.as<int32_t>(), rows, MaxI32(), c->nnz, st));
        heads.release();
        k_check_cols<<<grid_for(c->nnz), 256, 0, st>>>(rows, col_idx, c->nnz, c->n, bad.as<int>());
        TSMV_CUDA(cudaGetLastError());
        b = read1(bad.as<int>(), st);
        TSMV_REQUIRE(b == 0, "tsmv_create: column indices must be strictly ascending per row and < ncols");
        k_colcount<<<grid_for(c->nnz), 256, 0, st>>>(col_idx, c->nnz, c->outdeg.as<int32_t>());
    }
    TSMV_CUDA(cudaGetLastError());
    TSMV_CUDA(cudaStreamSynchronize(st));
}

void build_tileset(tsmv_ctx *c, TileSet &S, const int32_t *rows, const int32_t *cols, const void *vals,
                   int64_t nnz, int64_t dimR, int64_t dimC, bool want_vals, bool want_planes, cudaStream_t st,
                   const int32_t *hot_map) {
    int thr = c->opt.sparse_tile_max_nnz;
    S.hot_list = hot_map ? c->hot_list.as<int32_t>() : nullptr;
    bool f32 = c->dtype == TSMV_F32;
    const void *v = want_vals ? vals : nullptr;
#define TSMV_BUILD(NTV)                                                                                  \
    if (v && f32) build_nt<NTV, float>(S, rows, cols, (const float *)v, nnz, dimR, dimC, thr, want_planes, st, hot_map); \
    else build_nt<NTV, double>(S, rows, cols, (const double *)v, nnz, dimR, dimC, thr, want_planes, st, hot_map);
    switch (c->nt) {
        case 16: TSMV_BUILD(16); break;
        case 32: TSMV_BUILD(32); break;
        default: TSMV_BUILD(64); break;
    }
#undef TSMV_BUILD
}

__global__ void k_tilerow_nnz(const int32_t *__restrict__ indeg, int64_t m, int nt, int64_t nTR,
                              long long *__restrict__ out) {
    for (int64_t I = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; I < nTR; I += (int64_t)gridDim.x * blockDim.x) {
        long long s = 0;
        for (int64_t r = I * nt; r < (I + 1) * nt && r < m; ++r) s += indeg[r];
        out[I] = s;
    }
}

// Pick the tile rows whose rows are privatised in shared memory by the SpMSpV
// kernel: the HOT_SLOTS/nt tile rows with the most nonzeros (power-law hubs get
// thousands of same-address fp64 atomics per call otherwise).
void choose_hot_rows(tsmv_ctx *c, cudaStream_t st, DevBuf &hot_map) {
    const int nt = c->nt;
    const int64_t nTR = (c->m + nt - 1) / nt;
    const int K = (int)std::min<int64_t>(HOT_SLOTS / nt, nTR);
    c->n_hot = 0;
    if (K <= 0 || c->m == 0) return;
    DevBuf tr;
    tr.alloc(nTR * 8);
    k_tilerow_nnz<<<grid_for(nTR), 256, 0, st>>>(c->indeg.as<int32_t>(), c->m, nt, nTR, tr.as<long long>());
    TSMV_CUDA(cudaGetLastError());
    std::vector<long long> h(nTR);
    TSMV_CUDA(cudaMemcpyAsync(h.data(), tr.p, nTR * 8, cudaMemcpyDeviceToHost, st));
    TSMV_CUDA(cudaStreamSynchronize(st));
    std::vector<int32_t> idx(nTR);
    for (int64_t i = 0; i < nTR; ++i) idx[i] = (int32_t)i;
    std::partial_sort(idx.begin(), idx.begin() + K, idx.end(), [&](int32_t a, int32_t b) {
        return h[a] != h[b] ? h[a] > h[b] : a < b;
    });
    std::vector<int32_t> hot;
    for (int q = 0; q < K; ++q)
        if (h[idx[q]] >= 2 * nt) hot.push_back(idx[q]);  // only genuinely heavy tile rows
    c->n_hot = (int)hot.size();
    if (hot.empty()) return;
    std::vector<int32_t> map(nTR, -1);
    for (size_t q = 0; q < hot.size(); ++q) map[hot[q]] = (int32_t)q;
    c->hot_list.alloc(hot.size() * 4);
    TSMV_CUDA(cudaMemcpy(c->hot_list.p, hot.data(), hot.size() * 4, cudaMemcpyHostToDevice));
    hot_map.alloc(nTR * 4);
    TSMV_CUDA(cudaMemcpy(hot_map.p, map.data(), nTR * 4, cudaMemcpyHostToDevice));
}

bool same_pattern_transposed(tsmv_ctx *c, const int32_t *rows, const int32_t *cols, int64_t nnz, cudaStream_t st) {
    if (nnz == 0) return true;
    DevBuf a, b, bs, diff;
    CubTemp tmp;
    a.alloc(nnz * 8);
    b.alloc(nnz * 8);
    bs.alloc(nnz * 8);
    diff.alloc(4);
    TSMV_CUDA(cudaMemsetAsync(diff.p, 0, 4, st));
    k_keys_pattern<<<grid_for(nnz), 256, 0, st>>>(rows, cols, nnz, c->n, false, a.as<unsigned long long>());
    k_keys_pattern<<<grid_for(nnz), 256, 0, st>>>(rows, cols, nnz, c->n, true, b.as<unsigned long long>());
    size_t tb = 0;
    cub::DeviceRadixSort::SortKeys(nullptr, tb, b.as<unsigned long long>(), bs.as<unsigned long long>(), nnz, 0,
                                   64, st);
    cub::DeviceRadixSort::SortKeys(tmp.get(tb), tb, b.as<unsigned long long>(), bs.as<unsigned long long>(), nnz,
                                   0, 64, st);
    k_cmp<<<grid_for(nnz), 256, 0, st>>>(a.as<unsigned long long>(), bs.as<unsigned long long>(), nnz,
                                          diff.as<int>());
    TSMV_CUDA(cudaGetLastError());
    int d = read1(diff.as<int>(), st);
    return d == 0;
}

}  // namespace tsmv
