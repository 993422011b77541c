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
}  // namespace dts
