// K6 — RDG on the FP64 CUDA-core pipe (placeholder until the kernel lands).
#include <cuda_runtime.h>

#include "kernels.hpp"

namespace lora {
bool rdg2d_supported(const Plan&) { return false; }
cudaError_t launch_rdg2d(const Plan&, const double*, double*, cudaStream_t) { return cudaErrorNotSupported; }
}  // namespace lora
