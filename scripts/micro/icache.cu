// Microbenchmark: cost of executing N straight-line instructions once (cold
// instruction cache) vs a loop executing the same count from a small body.
#include <cstdio>
#include <cuda_runtime.h>
template <int N>
__global__ void k_straight(unsigned *out, unsigned seed) {
    unsigned x = seed + threadIdx.x;
#pragma unroll
    for (int i = 0; i < N; ++i) x = (x ^ (x >> 7)) * 2654435761u + (unsigned)i * 40503u;
    if (x == 0x12345u) out[0] = x;
}
__global__ void k_loop(unsigned *out, unsigned seed, int n) {
    unsigned x = seed + threadIdx.x;
#pragma unroll 1
    for (int i = 0; i < n; ++i) x = (x ^ (x >> 7)) * 2654435761u + (unsigned)i * 40503u;
    if (x == 0x12345u) out[0] = x;
}
__global__ void k_flush(float *w, long long n) {
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x) w[i] = 1.f;
}
template <int N> float run(unsigned *o, float *w, bool flush, int blocks) {
    cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
    float best = 1e9, ms;
    for (int r = 0; r < 5; ++r) {
        if (flush) k_flush<<<4096, 512>>>(w, (512ll << 20) / 4);
        cudaEventRecord(a);
        k_straight<N><<<blocks, 32>>>(o, r);
        cudaEventRecord(b); cudaEventSynchronize(b);
        cudaEventElapsedTime(&ms, a, b); best = ms < best ? ms : best;
    }
    return best * 1e3;
}
int main() {
    unsigned *o; float *w; cudaMalloc(&o, 64); cudaMalloc(&w, 512ll << 20);
    for (int fl = 0; fl < 2; ++fl)
        for (int blocks : {1, 148}) {
            printf("flush %d blocks %d: N=64 %.2f  N=1024 %.2f  N=2048 %.2f  N=4096 %.2f  N=8192 %.2f us\n", fl, blocks,
                   run<64>(o, w, fl, blocks), run<1024>(o, w, fl, blocks), run<2048>(o, w, fl, blocks),
                   run<4096>(o, w, fl, blocks), run<8192>(o, w, fl, blocks));
        }
    cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b); float ms;
    cudaEventRecord(a); k_loop<<<1, 32>>>(o, 1, 8192); cudaEventRecord(b); cudaEventSynchronize(b);
    cudaEventElapsedTime(&ms, a, b); printf("loop 8192 iters: %.2f us\n", ms * 1e3);
    printf("err %s\n", cudaGetErrorString(cudaGetLastError()));
}
