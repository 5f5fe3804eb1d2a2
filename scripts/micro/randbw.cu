// Microbenchmark: random-sector throughput of HBM on a cold L2 vs footprint
// (TLB reach) and memory-level parallelism.  Each thread issues R independent
// random loads of W bytes; total requests = threads * R.
#include <cstdio>
#include <cuda_runtime.h>
__device__ __forceinline__ unsigned long long mix(unsigned long long z) {
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}
__global__ void k_flush(float *w, long long n) {
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x) w[i] = 1.f;
}
template <int R, class T>
__global__ void k_rand(const T *p, long long nelem, long long seed, T *out) {
    long long t = blockIdx.x * (long long)blockDim.x + threadIdx.x;
    T acc = T();
    long long ix[R];
#pragma unroll
    for (int r = 0; r < R; ++r) ix[r] = (long long)(mix((t * R + r) * 0x9E3779B97F4A7C15ull + seed) % (unsigned long long)nelem);
    T v[R];
#pragma unroll
    for (int r = 0; r < R; ++r) v[r] = __ldcg(p + ix[r]);
#pragma unroll
    for (int r = 0; r < R; ++r) acc = acc ^ v[r];
    if (acc == (T)0x12345) out[0] = acc;
}
template <int R>
__global__ void k_red(double *p, long long nelem, long long seed) {
    long long t = blockIdx.x * (long long)blockDim.x + threadIdx.x;
#pragma unroll
    for (int r = 0; r < R; ++r) {
        long long ix = (long long)(mix((t * R + r) * 0x9E3779B97F4A7C15ull + seed) % (unsigned long long)nelem);
        atomicAdd(p + ix, 1.0);
    }
}
int main() {
    const long long MAXB = 4ll << 30;
    char *p; float *w; unsigned long long *out;
    cudaMalloc(&p, MAXB); cudaMalloc(&w, 512ll << 20); cudaMalloc(&out, 64);
    cudaMemset(p, 0, MAXB);
    cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
    float ms;
    auto flush = [&]() { k_flush<<<4096, 512>>>(w, (512ll << 20) / 4); };
    // empty baseline
    for (long long S : {64ll << 20, 256ll << 20, 1ll << 30, 4ll << 30}) {
        for (int threads : {1 << 18, 1 << 20}) {
            for (int R : {1, 4}) {
                float best = 1e9;
                for (int rep = 0; rep < 4; ++rep) {
                    flush();
                    cudaEventRecord(a);
                    int blocks = threads / 256;
                    if (R == 1) k_rand<1, unsigned><<<blocks, 256>>>((const unsigned *)p, S / 4, rep, (unsigned *)out);
                    else k_rand<4, unsigned><<<blocks, 256>>>((const unsigned *)p, S / 4, rep, (unsigned *)out);
                    cudaEventRecord(b); cudaEventSynchronize(b);
                    cudaEventElapsedTime(&ms, a, b);
                    best = ms < best ? ms : best;
                }
                double req = (double)threads * R;
                printf("u32 rand: footprint %5lld MB threads %8d R %d: %.2f us  -> %.1f G req/s\n", S >> 20, threads, R,
                       best * 1e3, req / (best * 1e-3) / 1e9);
            }
        }
    }
    for (long long S : {32ll << 20, 256ll << 20}) {
        for (int threads : {1 << 18, 1 << 20}) {
            float best = 1e9;
            for (int rep = 0; rep < 4; ++rep) {
                flush();
                cudaEventRecord(a);
                k_red<4><<<threads / 256, 256>>>((double *)p, S / 8, rep);
                cudaEventRecord(b); cudaEventSynchronize(b);
                cudaEventElapsedTime(&ms, a, b);
                best = ms < best ? ms : best;
            }
            double req = (double)threads * 4;
            printf("f64 RED rand: footprint %5lld MB reds %8.0f: %.2f us -> %.1f G red/s\n", S >> 20, req, best * 1e3,
                   req / (best * 1e-3) / 1e9);
        }
    }
    // warm L2 RED (no flush)
    for (int threads : {1 << 18, 1 << 20}) {
        float best = 1e9;
        for (int rep = 0; rep < 4; ++rep) {
            k_red<4><<<threads / 256, 256>>>((double *)p, (32ll << 20) / 8, rep);
            cudaEventRecord(a);
            k_red<4><<<threads / 256, 256>>>((double *)p, (32ll << 20) / 8, rep);
            cudaEventRecord(b); cudaEventSynchronize(b);
            cudaEventElapsedTime(&ms, a, b);
            best = ms < best ? ms : best;
        }
        double req = (double)threads * 4;
        printf("f64 RED warm-L2 32MB reds %8.0f: %.2f us -> %.1f G red/s\n", req, best * 1e3, req / (best * 1e-3) / 1e9);
    }
    printf("err %s\n", cudaGetErrorString(cudaGetLastError()));
}
