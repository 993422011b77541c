// Microbenchmark: cost of a 5-round warp argmin over (int64 S, int k) as in pop_batch.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
__global__ void k(const int64_t *in, long long *cyc, int *sink, int iters) {
    __shared__ int64_t req[32];
    if (threadIdx.x < 32) req[threadIdx.x] = in[threadIdx.x];
    __syncthreads();
    if (threadIdx.x < 32) {
        int acc = 0;
        long long t0 = clock64();
        for (int it = 0; it < iters; it++) {
            const int j = threadIdx.x;
            int kb = j < 4 ? j : -1;
            int64_t sb = j < 4 ? req[j] + it : INT64_MAX;
#pragma unroll
            for (int o = 16; o > 0; o >>= 1) {
                const int ko = __shfl_xor_sync(0xffffffffu, kb, o);
                const int64_t so = __shfl_xor_sync(0xffffffffu, sb, o);
                if (ko >= 0 && (kb < 0 || so < sb || (so == sb && ko < kb))) {
                    kb = ko;
                    sb = so;
                }
            }
            acc += kb;
            if (j == 0) req[it & 3] += 1;
        }
        long long t1 = clock64();
        if (threadIdx.x == 0) { cyc[0] = (t1 - t0) / iters; sink[0] = acc; }
    }
}
int main() {
    int64_t h[32]; for (int i = 0; i < 32; i++) h[i] = 1000 + 7 * i;
    int64_t *d; long long *c; int *s; cudaMalloc(&d, 256); cudaMallocManaged(&c, 8); cudaMalloc(&s, 8);
    cudaMemcpy(d, h, 256, cudaMemcpyHostToDevice);
    k<<<1, 128>>>(d, c, s, 10000); cudaDeviceSynchronize();
    printf("argmin 5 rounds: %lld cycles/iter\n", c[0]);
    k<<<1, 32>>>(d, c, s, 10000); cudaDeviceSynchronize();
    printf("argmin 5 rounds (1 warp CTA): %lld cycles/iter\n", c[0]);
}
