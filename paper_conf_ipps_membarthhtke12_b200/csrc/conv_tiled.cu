// conv_tiled.cu -- HBM-bound tiled convolution kernels (Gaussian / Sobel).
// First version: no tiled instance yet; the dispatcher uses conv_generic.
#include <cuda_runtime.h>

#include "kernels.h"

namespace lop {

bool conv_tiled_supported(const ConvGeneric &) { return false; }

cudaError_t launch_conv_tiled(const ConvGeneric &, cudaStream_t) { return cudaErrorNotSupported; }

}  // namespace lop
