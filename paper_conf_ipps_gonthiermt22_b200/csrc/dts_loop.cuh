// dts_loop.cuh -- launchers of the decision loop (see dts_loop.cu).
#pragma once
#include <cuda_runtime.h>

#include <cstdint>

#include "dts_internal.cuh"

namespace dts {
cudaError_t launch_init(const Inst *d_insts, int n_inst, uint64_t bw, int64_t work, cudaStream_t st);
// One CTA per instance (grid CTAs pull instances from *work_counter).
cudaError_t launch_loop(const Inst *d_insts, int n_inst, int block, int grid, int *work_counter,
                        int smem_bytes, cudaStream_t st);
// Task shards (§8(e)) of one instance on one device: n_inst CTAs that
// exchange inside the kernel, so a cooperative launch (all co-resident).
cudaError_t launch_loop_coop(const Inst *d_insts, int n_inst, int block, int *work_counter, int smem_bytes,
                             cudaStream_t st);
int loop_max_blocks_per_sm(int block, int smem_bytes);
int loop_static_smem();
// The same loop specialised at compile time (dts_loop_fast.cu) to row-derived
// state, one shard, W = 0 and DARTS+LUF (Inst::sl, G = 1, W = 0, policy LUF).
cudaError_t launch_loop_fast(const Inst *d_insts, int n_inst, int block, int grid, int *work_counter,
                             int smem_bytes, cudaStream_t st);
int loop_max_blocks_per_sm_fast(int block, int smem_bytes);
int loop_static_smem_fast();

// One WARP per instance (dts_warp.cu): small instances of the fast mode with
// <= 2 inputs per task.  Shared-memory slice of one instance (byte offsets),
// computed identically by the host (launch size) and the kernel.
struct WarpLayout {
    int nw, n4, n8;
    int resm, al, dp, u, hh, np, plan, rl;
    int64_t total;
};
__host__ __device__ inline WarpLayout warp_layout(int m, int n, int K, int pcap, int rcap) {
    WarpLayout L;
    L.nw = (n + 31) / 32 > 0 ? (n + 31) / 32 : 1;
    L.n4 = (n + 3) & ~3;
    L.n8 = (n + 7) & ~7;
    int64_t off = 0;
    auto put = [&](int64_t bytes) {
        const int64_t o = off;
        off += (bytes + 15) & ~int64_t(15);
        return (int)o;
    };
    L.resm = put(4ll * L.n4);  // per datum: bit k = resident on simulated GPU k
    L.al = put(4ll * (m / 32 + 1));
    L.dp = put(4ll * (n + 1));
    L.u = put(2ll * L.n8);
    L.hh = put(4ll * K * L.n4);
    L.np = put(2ll * K * L.n8);
    L.plan = put(4ll * K * pcap);
    L.rl = put(4ll * K * rcap);
    int64_t tot = off;
    if (L.np + 8ll * n > tot) tot = L.np + 8ll * n;  // build scratch (mask, cursor) over np..
    if (tot < 256) tot = 256;                          // result assembly's offsets
    L.total = tot;
    return L;
}
cudaError_t launch_warp(const Inst *d_insts, int n_inst, int grid, int *work_counter, int smem_bytes,
                        cudaStream_t st);
int warp_max_blocks_per_sm(int smem_bytes);
}  // namespace dts
