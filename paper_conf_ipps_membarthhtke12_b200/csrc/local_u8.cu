// local_u8.cu -- u8 -> i32 instances of the local operator over several
// accessors (local_impl.cuh).
#include "local_impl.cuh"

namespace lop {

cudaError_t launch_local_u8part(const LocalParams &p, bool tiled, cudaStream_t stream)
{
    return launch_local_u8<true>(p, tiled, stream);
}

}  // namespace lop
