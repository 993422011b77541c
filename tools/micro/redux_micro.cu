// Warp-wide 64-bit max: 5 xor-shuffle rounds vs two redux.sync (hi, then lo among the hi maxima).
#include <cstdio>
#include <cuda_runtime.h>

__device__ __forceinline__ unsigned long long max_shfl(unsigned long long v) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        unsigned long long t = __shfl_xor_sync(0xffffffffu, v, o);
        v = t > v ? t : v;
    }
    return v;
}
__device__ __forceinline__ unsigned long long max_redux(unsigned long long v) {
    const unsigned hi = (unsigned)(v >> 32), lo = (unsigned)v;
    const unsigned mh = __reduce_max_sync(0xffffffffu, hi);
    const unsigned ml = __reduce_max_sync(0xffffffffu, hi == mh ? lo : 0u);
    return ((unsigned long long)mh << 32) | ml;
}
__global__ void k(long long *out, int mode, int iters) {
    unsigned long long v = (unsigned long long)(threadIdx.x * 2654435761u) << 20 | threadIdx.x;
    long long t0 = clock64();
    if (mode == 0)
        for (int i = 0; i < iters; i++) v = max_shfl(v ^ i) + threadIdx.x;
    else if (mode == 1)
        for (int i = 0; i < iters; i++) v = max_redux(v ^ i) + threadIdx.x;
    else
        for (int i = 0; i < iters; i++) v = __reduce_add_sync(0xffffffffu, (unsigned)v ^ i) + threadIdx.x;
    long long t1 = clock64();
    if (threadIdx.x == 0) { out[0] = t1 - t0; out[1] = (long long)v; }
}
int main() {
    long long *d, h[2];
    cudaMalloc(&d, 16);
    const char *nm[] = {"64-bit max, 5 shfl rounds", "64-bit max, 2 redux", "32-bit add, 1 redux"};
    for (int m = 0; m < 3; m++) {
        k<<<1, 32>>>(d, m, 1000);
        k<<<1, 32>>>(d, m, 1000);
        cudaMemcpy(h, d, 16, cudaMemcpyDeviceToHost);
        printf("%-28s %6.1f cycles/op\n", nm[m], h[0] / 1000.0);
    }
}
