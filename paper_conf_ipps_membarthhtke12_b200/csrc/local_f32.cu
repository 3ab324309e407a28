// local_f32.cu -- f32 instances of the local operator over several accessors
// (local_impl.cuh) and the C-ABI-side dispatcher.
#include "local_impl.cuh"

namespace lop {

cudaError_t launch_local_u8part(const LocalParams &p, bool tiled, cudaStream_t stream);   // local_u8.cu

cudaError_t launch_local(const LocalParams &p, bool tiled, cudaStream_t stream)
{
    return p.u8 ? launch_local_u8part(p, tiled, stream) : launch_local_u8<false>(p, tiled, stream);
}

}  // namespace lop
