// Microbenchmark: cost of dependent random-load "hops" on a cold L2 (after a
// flush), launch overheads.  nvcc -gencode arch=compute_100a,code=sm_100a -O3 hops.cu -o hops
#include <cstdio>
#include <cuda_runtime.h>
#include <vector>
__global__ void k_init(unsigned *p, long long n, unsigned long long seed) {
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x) {
        unsigned long long z = (i + seed) * 0x9E3779B97F4A7C15ull;
        z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
        z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
        z ^= z >> 31;
        p[i] = (unsigned)(z % (unsigned long long)n);
    }
}
__global__ void k_flush(float *w, long long n) {
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x) w[i] = 1.f;
}
// every thread: H dependent loads starting at a thread-dependent index
template <int H>
__global__ void k_chain(const unsigned *p, long long n, unsigned *out, int active) {
    long long t = blockIdx.x * (long long)blockDim.x + threadIdx.x;
    if (t >= active) return;
    unsigned v = (unsigned)((t * 2654435761ull) % n);
#pragma unroll 1
    for (int h = 0; h < H; ++h) v = __ldcg(p + v);
    if (v == 0xffffffffu) out[0] = v;
}
__global__ void k_empty(int *o) { if (o && threadIdx.x == 9999) o[0] = 1; }
int main() {
    const long long N = 1ll << 28;  // 1 GiB of u32
    unsigned *p; float *w; unsigned *out;
    cudaMalloc(&p, N * 4); cudaMalloc(&w, 512ll << 20); cudaMalloc(&out, 64);
    k_init<<<4096, 256>>>(p, N, 12345);
    cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
    auto flush = [&]() { k_flush<<<4096, 512>>>(w, (512ll << 20) / 4); };
    float ms;
    for (int act : {1, 32, 148 * 32, 148 * 512, 148 * 2048}) {
        int blocks = (act + 511) / 512, th = act < 512 ? act : 512;
        for (int H : {1, 2, 4, 8}) {
            float best = 1e9;
            for (int rep = 0; rep < 5; ++rep) {
                flush();
                cudaEventRecord(a);
                switch (H) {
                case 1: k_chain<1><<<blocks, th>>>(p, N, out, act); break;
                case 2: k_chain<2><<<blocks, th>>>(p, N, out, act); break;
                case 4: k_chain<4><<<blocks, th>>>(p, N, out, act); break;
                default: k_chain<8><<<blocks, th>>>(p, N, out, act); break;
                }
                cudaEventRecord(b); cudaEventSynchronize(b);
                cudaEventElapsedTime(&ms, a, b);
                best = ms < best ? ms : best;
            }
            printf("cold chain: threads %7d hops %d: %.2f us total\n", act, H, best * 1e3);
        }
    }
    // same, L2-warm (no flush; 64 MB subset)
    for (int H : {1, 4, 8}) {
        float best = 1e9;
        for (int rep = 0; rep < 5; ++rep) {
            cudaEventRecord(a);
            if (H == 1) k_chain<1><<<1, 1>>>(p, 1 << 24, out, 1);
            else if (H == 4) k_chain<4><<<1, 1>>>(p, 1 << 24, out, 1);
            else k_chain<8><<<1, 1>>>(p, 1 << 24, out, 1);
            cudaEventRecord(b); cudaEventSynchronize(b);
            cudaEventElapsedTime(&ms, a, b);
            best = ms < best ? ms : best;
        }
        printf("warm-ish chain 1 thread hops %d: %.2f us\n", H, best * 1e3);
    }
    // empty launches
    for (int th : {32, 512}) {
        float best = 1e9;
        for (int rep = 0; rep < 10; ++rep) {
            flush();
            cudaEventRecord(a);
            k_empty<<<148, th>>>(nullptr);
            cudaEventRecord(b); cudaEventSynchronize(b);
            cudaEventElapsedTime(&ms, a, b);
            best = ms < best ? ms : best;
        }
        printf("empty launch 148x%d after flush: %.2f us\n", th, best * 1e3);
    }
    {
        float best = 1e9;
        for (int rep = 0; rep < 10; ++rep) {
            flush();
            cudaEventRecord(a);
            int *nil = nullptr; void *args[] = {&nil};
            cudaLaunchCooperativeKernel((void *)k_empty, 148, 512, args, 0, 0);
            cudaEventRecord(b); cudaEventSynchronize(b);
            cudaEventElapsedTime(&ms, a, b);
            best = ms < best ? ms : best;
        }
        printf("empty cooperative launch 148x512 after flush: %.2f us\n", best * 1e3);
    }
    printf("err %s\n", cudaGetErrorString(cudaGetLastError()));
}
