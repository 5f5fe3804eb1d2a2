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
#include "bfs_dev.cuh"

namespace tsmv {

namespace {

constexpr int BFB = 512;  // threads per CTA

struct BfsFusedArgs {
    BfsTiles P, Q;
    BfsView B;            // V, F (=F0), Fn (=F1), levels, n, m
    const int *outdeg, *indeg;
    ListsView Lv;
    long long *partials;  // [G][8]
    Counters *cnt;
    Counters *hm;         // mapped: fsize (levels), reached, edges
    int *dir_out;         // [max_levels]
    long long *front_out; // [max_levels]
    long long source, nnz, nseg, NW, nTR_local, max_levels;
    double alpha, dens;
    int force;
    unsigned long long bar_base;
    // resume / hand-off: the kernel stops before expanding a
    // Pull-CSC level when stop_on_pull is set; the host runs that level with the
    // high-occupancy per-level kernels and resumes the kernel afterwards
    int resume, stop_on_pull;
    long long level0, mu0, reached0, edges0;
};

template <int NT>
__device__ __forceinline__ void seg_counts(const BfsFusedArgs &a, const uint32_t *F, long long J, long long *v) {
    using word_t = typename Tr<NT>::word_t;
    const word_t bits = seg_bits<NT>(F, J);
    if (!bits) return;
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

template <int NT>
__global__ void __launch_bounds__(BFB, 1) k_bfs_fused(BfsFusedArgs a) {
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

    // ---- init: V = padding bits + source, F0 = {source}, F1 = 0, levels
    for (long long w = gtid; w < (a.resume ? 0 : a.NW); w += gthreads) {
        const long long v0 = w * 32;
        uint32_t pad = 0;
        if (v0 + 32 > B.n) pad = (v0 >= B.n) ? 0xffffffffu : (0xffffffffu << (B.n - v0));
        const uint32_t s = (a.source >= v0 && a.source < v0 + 32) ? (1u << (a.source - v0)) : 0u;
        B.V[w] = pad | s;
        Fa[w] = s;
        Fb[w] = 0;
    }
    if (!a.resume)
        for (long long v = gtid; v < B.m_local; v += gthreads) B.levels[v] = (v == a.source) ? 0 : -1;
    grid_sync(&a.cnt->bar, target);

    long long mu = a.resume ? a.mu0 : a.nnz, reached = a.reached0, edges = a.edges0;
    int stopped = 0;
    const long long S = (a.nseg + G - 1) / G;                 // segments per CTA
    const long long js0 = (long long)b * S, js1 = min(a.nseg, js0 + S);
    const long long per = (S + BFB - 1) / BFB;
    const long long tj0 = min(js1, js0 + tid * per), tj1 = min(js1, tj0 + per);
    int level = (int)a.level0;
    unsigned long long t_s1 = 0, t_s2 = 0, t_e = 0, tq = b == 0 && tid == 0 ? globaltimer_ns() : 0;
    for (; level < a.max_levels; ++level) {
        B.F = Fa;
        B.Fn = Fb;
        B.level = level;
        // ---- S: count this thread's segments, clear the consumed bitmap Fb
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
        if (tid < 32) {
            long long pre[8] = {0, 0, 0, 0, 0, 0, 0, 0}, all[8] = {0, 0, 0, 0, 0, 0, 0, 0};
            for (int g = lane; g < G; g += 32) {
#pragma unroll
                for (int i = 0; i < 7; ++i) {
                    const long long x = __ldcg(&a.partials[g * 8 + i]);
                    all[i] += x;
                    if (g < b) pre[i] += x;
                }
            }
#pragma unroll
            for (int i = 0; i < 7; ++i) {
#pragma unroll
                for (int o = 16; o > 0; o >>= 1) {
                    pre[i] += __shfl_xor_sync(0xffffffffu, pre[i], o);
                    all[i] += __shfl_xor_sync(0xffffffffu, all[i], o);
                }
            }
            if (lane == 0)
                for (int i = 0; i < 7; ++i) {
                    s_pre[i] = pre[i];
                    s_tot[i] = all[i];
                }
        }
        __syncthreads();
        const long long fsize = s_tot[4], mf = s_tot[5];
        mu -= s_tot[6];
        if (fsize == 0) break;
        reached += fsize;
        edges += mf;
        const int dir = choose_dir_dev(a.force, a.alpha, a.dens, B.n, fsize, mf, mu);
        if (b == 0 && tid == 0) {
            a.dir_out[level] = dir;
            a.front_out[level] = fsize;
        }
        if (dir == TSMV_DIR_PULL_CSC && a.stop_on_pull) {
            stopped = 1;  // uniform across CTAs: same totals, same decision
            break;
        }
        // lists (Push-CSC needs both, Push-CSR the side list; pull none)
        if (dir != TSMV_DIR_PULL_CSC) {
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
                    write_chunks(a.Lv.Ct, oWt, wt, (int)oLt);
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
                        write_chunks(a.Lv.Cs, oWs, ws, (int)oLs);
                        ++oLs;
                        oWs += ws;
                    }
                }
            }
            if (b == G - 1 && tid == 0) {
                a.Lv.Lt_wpre[s_tot[0]] = s_tot[1];
                a.Lv.Ls_wpre[s_tot[2]] = s_tot[3];
            }
        }
        grid_sync(&a.cnt->bar, target);
        if (b == 0 && tid == 0) {
            const unsigned long long t = globaltimer_ns();
            t_s2 += t - tq;
            tq = t;
        }

        // ---- E: expand
        if (dir == TSMV_DIR_PULL_CSC) {
            for (long long I = gwarp; I < a.nTR_local; I += gwarps) pull_rowtile<NT>(a.Q, B, I, lane);
            for (long long u = gtid; u < B.m_local; u += gthreads) pull_side_vertex<NT>(a.Q, B, u);
        } else {
            if (dir == TSMV_DIR_PUSH_CSR)
                for (long long t = gtid; t < a.Q.T; t += gthreads) push_csr_item<NT>(a.Q, B, t);
            const long long nLt = s_tot[0], Wt = s_tot[1], nLs = s_tot[2], Ws = s_tot[3];
            const long long nCt = dir == TSMV_DIR_PUSH_CSC ? (Wt + CHUNK - 1) >> CHUNK_LOG : 0;
            const long long nCs = (Ws + CHUNK - 1) >> CHUNK_LOG;
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
                                               (word_t)__ldcg(&a.Lv.Lt_mask[s]));
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
                            push_side_item<NT>(a.P, B, __ldcg(&a.Lv.Ls_beg[s0 + q]) + (i - win[q]));
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
        a.hm->nLt = (Fa == a.B.F) ? 0 : 1;  // which bitmap holds the current frontier
        a.hm->Wt = (long long)t_s1;  // phase times (ns, CTA 0): count, lists, expand
        a.hm->nLs = (long long)t_s2;
        a.hm->Ws = (long long)t_e;
    }
}

}  // namespace

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

// Launch the fused kernel from `level0` (resume) on bitmaps (Fa, Fb).  Returns
// true if it stopped before a Pull-CSC level.
bool bfs_fused_launch(tsmv_ctx *c, long long source, cudaStream_t st, bool resume, long long level0, uint32_t *Fa,
                      uint32_t *Fb, long long mu, long long reached, long long edges, bool stop_on_pull,
                      long long max_levels, long long &level_out, long long &mu_out, long long &reached_out,
                      long long &edges_out, int &cur_out) {
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
    a.source = source;
    a.nnz = c->nnz;
    a.nseg = c->nTC;
    a.NW = (long long)(c->V.bytes / 4);
    a.nTR_local = (c->m + c->nt - 1) / c->nt;
    a.max_levels = max_levels;
    a.alpha = c->opt.pull_alpha;
    a.dens = c->opt.push_csr_density;
    a.force = c->opt.force_dir;
    a.bar_base = c->bar_base;
    a.resume = resume ? 1 : 0;
    a.stop_on_pull = stop_on_pull ? 1 : 0;
    a.level0 = level0;
    a.mu0 = mu;
    a.reached0 = reached;
    a.edges0 = edges;
    void *args[] = {&a};
    void *f = c->nt == 16 ? (void *)k_bfs_fused<16> : c->nt == 32 ? (void *)k_bfs_fused<32> : (void *)k_bfs_fused<64>;
    const int G = c->bfs_blocks;
    TSMV_CUDA(cudaLaunchCooperativeKernel(f, dim3(G), dim3(BFB), args, 0, st));
    TSMV_CUDA(cudaStreamSynchronize(st));
    volatile Counters *h = c->hcnt;
    const long long L = h->fsize;
    const bool stopped = h->din != 0;
    level_out = L;
    reached_out = h->reached;
    edges_out = h->edges;
    mu_out = h->mf;
    cur_out = (int)h->nLt;
    // barriers: 1 (init) + 3 per expanded level + 1 for the final scan (empty frontier or pull stop)
    const long long expanded = L - level0;
    const long long nbar = 1 + 3 * expanded + ((L < max_levels) ? 1 : 0);
    c->bar_base += (unsigned long long)nbar * (unsigned long long)G;
    return stopped;
}

}  // namespace tsmv
