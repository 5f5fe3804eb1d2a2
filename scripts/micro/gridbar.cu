// Microbenchmark: cost of one grid barrier (cooperative launch, 1 CTA / SM) for
// several barrier implementations.  nvcc -arch=sm_100a -O3 gridbar.cu -o gridbar
#include <cstdio>
#include <cuda_runtime.h>
__device__ __forceinline__ unsigned long long ld_acq(const unsigned long long *p) {
    unsigned long long v;
    asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
template <int MODE>
__global__ void k(unsigned long long *bar, int iters, int sleepns) {
    unsigned long long target = 0;
    for (int i = 0; i < iters; ++i) {
        __syncthreads();
        target += gridDim.x;
        if (threadIdx.x == 0) {
            __threadfence();
            if (MODE == 0) atomicAdd(bar, 1ull);
            else asm volatile("red.release.gpu.global.add.u64 [%0], 1;" ::"l"(bar) : "memory");
            while (ld_acq(bar) < target) {
                if (sleepns) __nanosleep(sleepns);
            }
            __threadfence();
        }
        __syncthreads();
    }
}
int main() {
    int sms;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    unsigned long long *bar;
    cudaMalloc(&bar, 8);
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    for (int mode = 0; mode < 2; ++mode)
        for (int threads : {256, 512, 1024})
            for (int sl : {0, 20, 100}) {
                int iters = 1000;
                void *args[] = {&bar, &iters, &sl};
                for (int rep = 0; rep < 2; ++rep) {
                    cudaMemset(bar, 0, 8);
                    cudaEventRecord(a);
                    cudaLaunchCooperativeKernel(mode == 0 ? (void *)k<0> : (void *)k<1>, sms, threads, args, 0, 0);
                    cudaEventRecord(b);
                    cudaEventSynchronize(b);
                    float ms;
                    cudaEventElapsedTime(&ms, a, b);
                    if (rep) printf("mode %d threads %4d sleep %3d: %.3f us per barrier\n", mode, threads, sl, ms * 1e3 / iters);
                }
            }
    // empty kernel launch cost
    cudaEventRecord(a);
    for (int i = 0; i < 100; ++i) {
        int it = 0, sl = 0;
        void *args[] = {&bar, &it, &sl};
        cudaLaunchCooperativeKernel((void *)k<0>, sms, 512, args, 0, 0);
    }
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms;
    cudaEventElapsedTime(&ms, a, b);
    printf("empty cooperative launch (back to back): %.3f us\n", ms * 10);
    printf("err %s\n", cudaGetErrorString(cudaGetLastError()));
}
