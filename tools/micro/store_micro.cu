// One thread: the sequential pop loop's pattern -- T from shared memory, then
// four global stores at T-dependent addresses (+ 2 shared stores) per iteration.
#include <cstdio>
#include <cuda_runtime.h>

__global__ void k(long long *out, long long *ts, long long *te, int *sg, int *stk, int mode, int iters) {
    __shared__ int pl[4096];
    __shared__ long long last[4];
    for (int i = threadIdx.x; i < 4096; i += blockDim.x) pl[i] = (i * 2654435761u) % 100000;
    __syncthreads();
    if (threadIdx.x) return;
    long long g = 0, mk = 0;
    long long t0 = clock64();
    for (int h = 0; h < iters; h++) {
        const int T = pl[h & 4095];
        const long long st = g > h ? g : h, en = st + 534059;
        g = en;
        if (mode == 0) {         // __stcg
            __stcg(&ts[T], st); __stcg(&te[T], en); __stcg(&sg[h], 1); __stcg(&stk[h], T);
        } else if (mode == 1) {  // plain stores
            ts[T] = st; te[T] = en; sg[h] = 1; stk[h] = T;
        } else if (mode == 2) {  // no global stores
            mk += T;
        } else {                 // plain stores + shared stores
            ts[T] = st; te[T] = en; sg[h] = 1; stk[h] = T; last[0] = T; last[1] = en;
        }
        mk = en > mk ? en : mk;
    }
    long long t1 = clock64();
    out[0] = t1 - t0;
    out[1] = mk + g;
}
int main() {
    long long *d, h[2], *ts, *te;
    int *sg, *stk;
    cudaMalloc(&d, 16); cudaMalloc(&ts, 8 * 100000); cudaMalloc(&te, 8 * 100000);
    cudaMalloc(&sg, 4 * 100000); cudaMalloc(&stk, 4 * 100000);
    const char *nm[] = {"4x __stcg", "4x plain st", "no global st", "4x st + 2 sts"};
    for (int m = 0; m < 4; m++) {
        k<<<1, 128>>>(d, ts, te, sg, stk, m, 20000);
        k<<<1, 128>>>(d, ts, te, sg, stk, m, 20000);
        cudaMemcpy(h, d, 16, cudaMemcpyDeviceToHost);
        printf("%-16s %6.1f cycles/iter\n", nm[m], h[0] / 20000.0);
    }
}
