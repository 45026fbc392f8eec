// k_gemm_tc.cu — tcgen05 3xTF32 GEMM (placeholder until the tensor-core path
// lands; the SIMT path in k_gemm.cu serves every shape meanwhile).
#include <cuda_runtime.h>
#include <stdint.h>

#include "gnn_internal.h"

namespace gnn {

cudaError_t launch_gemm_tc(const float *, int64_t, const float *, int64_t, float *, int64_t, int64_t,
                           int32_t, int32_t, const float *, const float *, int32_t, cudaStream_t) {
  return cudaErrorNotSupported;
}

}  // namespace gnn
