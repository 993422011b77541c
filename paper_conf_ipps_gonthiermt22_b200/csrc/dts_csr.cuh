// dts_csr.cuh -- device CSR build (§8(a) a1), see dts_csr.cu.
#pragma once
#include <cuda_runtime.h>

#include <cstddef>
#include <cstdint>

namespace dts {
size_t csr_scratch_bytes(int32_t m, int32_t n, int64_t E_raw);
cudaError_t build_csr(const int64_t *raw_ptr, const int32_t *raw_dat, int32_t m, int32_t n,
                      int64_t E_raw, int64_t *tptr, int32_t *tdat, int64_t *dptr, int32_t *ddat,
                      int4 *dedge, void *scratch, cudaStream_t st, int32_t t_lo, int32_t t_hi);
}  // namespace dts
