// cnn_fp32.cu -- CNN offload units U1, U2, U3 (placeholder until the FFMA kernels land).
#include "kernels.h"

namespace tg {
cudaError_t launch_cnn_u1(const CnnU1Args&, cudaStream_t) { return cudaErrorNotSupported; }
cudaError_t launch_cnn_u2(const CnnU2Args&, cudaStream_t) { return cudaErrorNotSupported; }
cudaError_t launch_cnn_u3(const CnnU3Args&, cudaStream_t) { return cudaErrorNotSupported; }
}  // namespace tg
