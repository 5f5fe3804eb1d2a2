// Microbenchmark (round 2): the fixed costs an SpMSpV call at T cannot avoid.
//  1. empty kernel between two CUDA events: no flush / write-only flush / write+read flush,
//     1x32 and 148x1024 (+ 100 KB dynamic smem, cooperative)
//  2. dependent random-load chains, cold, with T-like parallelism (42 K threads)
//  3. the same chains when the next hop was bulk-prefetched into L2
//     (cp.async.bulk.prefetch.L2) one hop earlier
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 floor.cu -o floor
#include <cstdio>
#include <cuda_runtime.h>

__global__ void k_init(unsigned *p, long long n, unsigned long long seed) {
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x) {
        unsigned long long z = (i + seed) * 0x9E3779B97F4A7C15ull;
        z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
        z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
        z ^= z >> 31;
        p[i] = (unsigned)(z % (unsigned long long)n) & ~63u;  // 256-byte aligned targets
    }
}
__global__ void k_write(float *w, long long n) {
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x) w[i] = 1.f;
}
__global__ void k_read(const float *r, long long n, float *o) {
    float s = 0;
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x) s += r[i];
    if (s == 123.f) o[0] = s;
}
__global__ void k_empty(int *o) { if (o && threadIdx.x == 9999) o[0] = 1; }
__global__ void k_empty_smem(int *o) {
    extern __shared__ int sm[];
    if (o && threadIdx.x == 9999) { sm[0] = 1; o[0] = sm[threadIdx.x & 7]; }
}

__device__ __forceinline__ void pf_l2(const void *p, unsigned bytes) {
    asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(p), "r"(bytes) : "memory");
}
__device__ __forceinline__ void pf1(const void *p) { asm volatile("prefetch.global.L2 [%0];" ::"l"(p)); }

// H dependent hops.  MODE 0: one load per hop.  MODE 1: a 256-byte run (16
// loads) per hop, the next target in its first word.  MODE 3: per hop, first an
// unrelated cold load, then the run (made dependent on it).  MODE 4: as 3, but the
// run is bulk-prefetched into L2 before the unrelated load is issued (one hop of
// lead: does the run then cost an L2 hop instead of a DRAM hop?).
template <int MODE>
__global__ void k_chain(const unsigned *p, long long n, unsigned *out, int active, int H) {
    long long t = blockIdx.x * (long long)blockDim.x + threadIdx.x;
    if (t >= active) return;
    unsigned v = (unsigned)((t * 2654435761ull) % n) & ~63u;
    unsigned acc = 0;
#pragma unroll 1
    for (int h = 0; h < H; ++h) {
        if (MODE == 0) {
            v = __ldcg(p + v);
        } else {
            const unsigned *q = p + v;
            if (MODE >= 3) {
                if (MODE == 4) pf_l2(q, 256);
                const unsigned x = __ldcg(p + ((v * 2654435761u + 977u) % (unsigned)n));
                q += (x == 0xffffffffu) ? 64 : 0;
            }
            unsigned nv = __ldcg(q);
            unsigned s = 0;
#pragma unroll
            for (int i = 1; i < 16; ++i) s += __ldcg(q + 4 * i);
            acc += s;
            v = nv;
        }
    }
    if ((v ^ acc) == 0xffffffffu) out[0] = v;
}

int main() {
    const long long N = 1ll << 28;  // 1 GiB of u32
    unsigned *p; float *w, *r; unsigned *out;
    cudaMalloc(&p, N * 4); cudaMalloc(&w, 256ll << 20); cudaMalloc(&r, 256ll << 20); cudaMalloc(&out, 64);
    cudaMemset(r, 0, 256ll << 20);
    k_init<<<4096, 256>>>(p, N, 12345);
    cudaFuncSetAttribute(k_empty_smem, cudaFuncAttributeMaxDynamicSharedMemorySize, 100 * 1024);
    cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
    auto flushw = [&]() { k_write<<<148 * 4, 1024>>>(w, (256ll << 20) / 4); };
    auto flushwr = [&]() { flushw(); k_read<<<148 * 4, 1024>>>(r, (256ll << 20) / 4, (float *)out); };
    float ms;
    const char *fl[3] = {"no flush", "write flush", "write+read flush"};
    for (int f = 0; f < 3; ++f) {
        for (int kind = 0; kind < 3; ++kind) {
            float best = 1e9, sum = 0;
            for (int rep = 0; rep < 20; ++rep) {
                if (f == 1) flushw();
                if (f == 2) flushwr();
                cudaEventRecord(a);
                if (kind == 0) k_empty<<<1, 32>>>(nullptr);
                else if (kind == 1) k_empty_smem<<<148, 1024, 100 * 1024>>>(nullptr);
                else {
                    int *nil = nullptr; void *args[] = {&nil};
                    cudaLaunchCooperativeKernel((void *)k_empty_smem, 148, 1024, args, 100 * 1024, 0);
                }
                cudaEventRecord(b); cudaEventSynchronize(b);
                cudaEventElapsedTime(&ms, a, b);
                best = ms < best ? ms : best;
                sum += ms;
            }
            printf("empty %-28s %-18s min %.2f us mean %.2f us\n",
                   kind == 0 ? "1x32" : kind == 1 ? "148x1024 100KB smem" : "coop 148x1024 100KB smem", fl[f],
                   best * 1e3, sum / 20 * 1e3);
        }
    }
    for (int act : {4096, 42000, 148 * 1024}) {
        for (int mode : {0, 1, 3, 4})
            for (int H : {1, 2, 4, 8}) {
                float best = 1e9;
                for (int rep = 0; rep < 5; ++rep) {
                    flushwr();
                    cudaEventRecord(a);
                    int blocks = (act + 255) / 256;
                    if (mode == 0) k_chain<0><<<blocks, 256>>>(p, N, out, act, H);
                    else if (mode == 1) k_chain<1><<<blocks, 256>>>(p, N, out, act, H);
                    else if (mode == 3) k_chain<3><<<blocks, 256>>>(p, N, out, act, H);
                    else k_chain<4><<<blocks, 256>>>(p, N, out, act, H);
                    cudaEventRecord(b); cudaEventSynchronize(b);
                    cudaEventElapsedTime(&ms, a, b);
                    best = ms < best ? ms : best;
                }
                printf("cold chain threads %6d mode %d (%s) hops %d: %.2f us\n", act, mode,
                       mode == 0 ? "1 load/hop" : mode == 1 ? "256B run/hop" : mode == 3 ? "cold load + run" : "cold load + run, run prefetched", H,
                       best * 1e3);
            }
    }
    printf("err %s\n", cudaGetErrorString(cudaGetLastError()));
}
