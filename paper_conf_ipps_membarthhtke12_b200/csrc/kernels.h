// kernels.h -- launchers implemented in the .cu files, called by lop_api.cpp.
#pragma once
#include <cuda_runtime.h>

#include "lop_params.h"

namespace lop {

cudaError_t launch_bilateral_generic(const BilateralGeneric &p, cudaStream_t stream);
cudaError_t launch_bilateral_tiled(const BilateralTiled &p, cudaStream_t stream);
cudaError_t launch_bilateral_sep(const BilateralSep &p, cudaStream_t stream);
cudaError_t launch_bilateral_pair(const BilateralSep &p, cudaStream_t stream);
int bilateral_sep_max_npoly(int rx);
cudaError_t launch_conv_generic(const ConvGeneric &p, cudaStream_t stream);
// Tiled convolution; returns cudaErrorNotSupported when no instance matches
// (the caller then falls back to the generic kernel).
cudaError_t launch_conv_tiled(const ConvGeneric &p, cudaStream_t stream);
bool conv_tiled_supported(const ConvGeneric &p);
// Exact separable factorisation (false if the mask is not rank 1 / too large).
bool conv_factor(const ConvGeneric &p, ConvSep &s);
// Local MIN / MAX over a mask domain (reduce.cu): tiled separable kernel for
// full windows up to 9x9, generic kernel otherwise.
cudaError_t launch_reduce(const ReduceParams &p, bool allow_tiled, cudaStream_t stream);
// Two local operators combined by a point operator (conv_pair.cu); the tiled
// launcher returns cudaErrorNotSupported when no instance matches.
cudaError_t launch_conv_pair(const ConvPair &p, cudaStream_t stream);
cudaError_t launch_conv_pair_generic(const ConvPairGeneric &p, cudaStream_t stream);
// Global SUM / MIN / MAX (global_reduce.cu): two launches (parts, final).
cudaError_t launch_global_reduce(const GlobalReduce &p, cudaStream_t stream);
// Fused two-stage convolution; cudaErrorNotSupported if no instance matches.
cudaError_t launch_conv_chain(const ConvChain &p, cudaStream_t stream);

// Local operator over several accessors (local.cu): tiled (shared-memory
// staging) or generic; the CTA shape from Algorithm 2 (select.cpp).
cudaError_t launch_local(const LocalParams &p, bool tiled, cudaStream_t stream);

// Laplacian-pyramid REDUCE and EXPAND (+ addend) (pyramid.cu).
cudaError_t launch_pyr_reduce(const PyrParams &p, cudaStream_t stream);
cudaError_t launch_pyr_expand(const PyrParams &p, cudaStream_t stream);

}  // namespace lop
