// Latency of shared-memory accesses through generic pointers (LD.E / ATOM.E)
// vs shared-space instructions (LDS / ATOMS / RED.shared), one thread, dependent chains.
#include <cstdio>
#include <cuda_runtime.h>

__device__ int *g_sink;

__global__ void k(long long *out, int *gptr_host_visible, int mode, int iters) {
    __shared__ int sm[1024];
    for (int i = threadIdx.x; i < 1024; i += blockDim.x) sm[i] = (i * 7 + 3) & 1023;
    __syncthreads();
    if (threadIdx.x != 0) return;
    int *gp = (mode & 1) ? sm : gptr_host_visible;  // runtime choice: generic pointer
    volatile int *vg = gp;
    int x = 1;
    long long t0 = clock64();
    switch (mode >> 1) {
        case 0:  // dependent generic load
            for (int i = 0; i < iters; i++) x = vg[x & 1023];
            break;
        case 1:  // dependent LDS
            for (int i = 0; i < iters; i++) x = ((volatile int *)sm)[x & 1023];
            break;
        case 2:  // generic atomic, result used
            for (int i = 0; i < iters; i++) x = atomicAdd(gp + (x & 1023), 1) & 1023;
            break;
        case 3:  // shared atomic, result used
            for (int i = 0; i < iters; i++) x = atomicAdd(sm + (x & 1023), 1) & 1023;
            break;
        case 4:  // generic atomic, result unused, then a dependent generic load
            for (int i = 0; i < iters; i++) { atomicAdd(gp + (x & 1023), 1); x = vg[(x + 1) & 1023]; }
            break;
        case 5:  // red.shared via cvta, then dependent LDS
            for (int i = 0; i < iters; i++) {
                unsigned a = (unsigned)__cvta_generic_to_shared(sm + (x & 1023));
                asm volatile("red.shared.add.s32 [%0], %1;" ::"r"(a), "r"(1) : "memory");
                x = ((volatile int *)sm)[(x + 1) & 1023];
            }
            break;
        case 6:  // generic store then generic load (store-to-load through generic)
            for (int i = 0; i < iters; i++) { vg[x & 1023] = i; x = vg[(x + 5) & 1023] & 1023; }
            break;
    }
    long long t1 = clock64();
    out[0] = t1 - t0;
    out[1] = x;
}

int main() {
    long long *d, h[2];
    int *gbuf;
    cudaMalloc(&d, 16);
    cudaMalloc(&gbuf, 4096);
    cudaMemset(gbuf, 0, 4096);
    const char *names[] = {"generic LD (smem)", "LDS", "generic ATOM used (smem)", "ATOMS used",
                           "generic ATOM unused + generic LD", "RED.shared + LDS", "generic ST + LD"};
    const int iters = 4096;
    for (int m = 0; m < 7; m++) {
        int mode = (m << 1) | 1;  // smem target
        k<<<1, 32>>>(d, gbuf, mode, iters);
        k<<<1, 32>>>(d, gbuf, mode, iters);
        cudaMemcpy(h, d, 16, cudaMemcpyDeviceToHost);
        printf("%-36s %7.1f cycles/iter\n", names[m], (double)h[0] / iters);
    }
    k<<<1, 32>>>(d, gbuf, (2 << 1) | 0, iters);
    k<<<1, 32>>>(d, gbuf, (2 << 1) | 0, iters);
    cudaMemcpy(h, d, 16, cudaMemcpyDeviceToHost);
    printf("%-36s %7.1f cycles/iter\n", "generic ATOM used (global)", (double)h[0] / iters);
    return 0;
}
