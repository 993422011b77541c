// Calibration: CTA barrier round trips and short smem loops, 128 threads.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
__device__ __forceinline__ void cta_sync() { __syncthreads(); __syncwarp(); }
template <int MODE>
__global__ void k(long long *cyc, int *sink, int iters) {
    __shared__ long long a[256];
    __shared__ int b[256];
    for (int i = threadIdx.x; i < 256; i += blockDim.x) { a[i] = i * 3; b[i] = i & 3; }
    cta_sync();
    long long t0 = clock64();
    int acc = 0;
    for (int it = 0; it < iters; it++) {
        if (MODE >= 1) cta_sync();
        if (MODE >= 2) cta_sync();
        if (MODE >= 3) {  // 12-entry counting loop
            const long long r = a[threadIdx.x & 15];
            int pos = 0;
            for (int q = 0; q < 12; q++) pos += (a[q] < r) || (a[q] == r && b[q] < 2);
            acc += pos;
        }
        if (MODE >= 4 && threadIdx.x == 0) {  // 10 dependent smem RMW on thread 0
            for (int q = 0; q < 10; q++) a[(acc + q) & 255] += acc;
        }
    }
    long long t1 = clock64();
    if (threadIdx.x == 0) { cyc[MODE] = (t1 - t0) / iters; sink[0] = acc; }
}
int main() {
    long long *c; int *s; cudaMallocManaged(&c, 64); cudaMalloc(&s, 8);
    k<1><<<1, 128>>>(c, s, 10000); k<2><<<1, 128>>>(c, s, 10000); k<3><<<1, 128>>>(c, s, 10000); k<4><<<1, 128>>>(c, s, 10000);
    cudaDeviceSynchronize();
    printf("1 cta_sync: %lld | 2 cta_sync: %lld | +12-count loop: %lld | +thread0 10 RMW: %lld cycles/iter\n", c[1], c[2], c[3], c[4]);
    k<2><<<1, 512>>>(c, s, 10000); cudaDeviceSynchronize();
    printf("512 threads, 2 cta_sync: %lld\n", c[2]);
}
