// Microbenchmark: cost of the thread-0 pop chain (smem plan entry + np RMW +
// scattered global stores) under variants.  nvcc -arch=sm_100a pop_micro.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

template <int MODE>
__global__ void k(int4 *gplan, int64_t *tst, int64_t *ten, int32_t *sg, int32_t *stk, int n_iter,
                  long long *cyc, int *sink) {
    __shared__ int4 pl[1024];
    __shared__ int np[4096];
    for (int i = threadIdx.x; i < 1024; i += blockDim.x) pl[i] = gplan[i];
    for (int i = threadIdx.x; i < 4096; i += blockDim.x) np[i] = 0;
    __syncthreads();
    if (threadIdx.x == 0) {
        int4 *P = (MODE & 4) ? gplan : pl;  // generic pointer
        int *N = np;
        long long t0 = clock64();
        int64_t req = 0, gfree = 0;
        int h = 0;
        for (int it = 0; it < n_iter; it++) {
            int4 e = P[h & 1023];
            h++;
            if (MODE & 1) {
                N[e.y & 4095] -= 1;
                N[e.z & 4095] -= 1;
            }
            if (MODE & 8) {  // generic atomics to smem
                atomicAdd(N + (e.y & 4095), 1);
                atomicAdd(N + (e.z & 4095), 1);
            }
            if (MODE & 16) {  // explicit shared atomics
                atomicAdd(&np[e.y & 4095], 1);
                atomicAdd(&np[e.z & 4095], 1);
            }
            int64_t start = req > gfree ? req : gfree;
            int64_t end = start + 17;
            gfree = end;
            if (MODE & 2) {
                tst[e.x] = start;
                ten[e.x] = end;
                sg[it] = 1;
                stk[it] = e.x;
            }
            req = end;
        }
        cyc[MODE] = (clock64() - t0) / n_iter;
        sink[0] = (int)req + N[5];
    }
}

int main() {
    const int NI = 100000;
    int4 *gplan; int64_t *tst, *ten; int32_t *sg, *stk; long long *cyc; int *sink;
    cudaMalloc(&gplan, 1024 * 16); cudaMalloc(&tst, 8 * 1048576); cudaMalloc(&ten, 8 * 1048576);
    cudaMalloc(&sg, 4 * NI); cudaMalloc(&stk, 4 * NI); cudaMallocManaged(&cyc, 8 * 32); cudaMalloc(&sink, 64);
    int4 h[1024];
    for (int i = 0; i < 1024; i++) h[i] = make_int4((i * 7919) % 1048576, i % 200, (i * 3) % 200 + 200, -1);
    cudaMemcpy(gplan, h, sizeof h, cudaMemcpyHostToDevice);
    k<0><<<1, 128>>>(gplan, tst, ten, sg, stk, NI, cyc, sink);
    k<1><<<1, 128>>>(gplan, tst, ten, sg, stk, NI, cyc, sink);
    k<2><<<1, 128>>>(gplan, tst, ten, sg, stk, NI, cyc, sink);
    k<3><<<1, 128>>>(gplan, tst, ten, sg, stk, NI, cyc, sink);
    k<7><<<1, 128>>>(gplan, tst, ten, sg, stk, NI, cyc, sink);
    k<8><<<1, 128>>>(gplan, tst, ten, sg, stk, NI, cyc, sink);
    k<16><<<1, 128>>>(gplan, tst, ten, sg, stk, NI, cyc, sink);
    cudaDeviceSynchronize();
    printf("cycles/iter: base %lld | +np RMW %lld | +4 global stores %lld | both %lld | both, plan in gmem %lld\n",
           cyc[0], cyc[1], cyc[2], cyc[3], cyc[7]);
    printf("generic atomics smem %lld | shared atomics %lld\n", cyc[8], cyc[16]);
    return 0;
}
