// sgemm_tf32.cu -- grouped SGEMM on tcgen05 TF32 tensor cores (placeholder launcher).
// The kernel is registered as unsupported until the tcgen05 path lands; the launcher
// fails loudly rather than falling back to anything else.
#include "../launch.h"

namespace svp {

cudaError_t launch_sgemm_tf32(const GemmDesc*, int, const void*, uint32_t, int, cudaStream_t) {
    return cudaErrorNotSupported;
}

}  // namespace svp
