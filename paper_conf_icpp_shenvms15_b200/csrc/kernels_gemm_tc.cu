// tcgen05 3xTF32 SGEMM (placeholder until the tensor-core path lands).
#include "kernels.h"

namespace mm {

cudaError_t sgemm_tf32x3_rows(const float*, const float*, float*, int64_t, int64_t, int64_t, int64_t,
                              int64_t, cudaStream_t, int) {
  return cudaErrorNotSupported;
}

}  // namespace mm
