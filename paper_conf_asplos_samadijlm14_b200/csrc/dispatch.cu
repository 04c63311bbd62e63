// dispatch.cu -- picks the kernel variant for a plan and an image layout.
#include "internal.h"

namespace ppx {

cudaError_t launch_generic(const Plan& p, const float* in, const View& v, float* out, long long opitch,
                           long long ofs, cudaStream_t s);

cudaError_t launch_stencil(const Plan& p, const float* in, const View& v, float* out, long long opitch,
                           long long ofs, cudaStream_t s) {
    return launch_generic(p, in, v, out, opitch, ofs, s);
}

}  // namespace ppx
