// arcv_k1_s3_dtu8.cu -- K1 with 3 stages, min 2 CTAs per SM, specialised for
// ARC_U8 regions (single-region calls: only that dtype's tile evaluation is
// compiled in, so the kernel is ~5x smaller); arcv_kernels.h.
#include <cuda_runtime.h>

#include "arcv_device.cuh"
#include "arcv_kernels.h"

namespace arcv {

KernelFnN<1> k1_s3_1_u8(bool xf) {
    return xf ? arcv_stream_kernel<3, 2, 1, true, (1 << ARC_U8)> : arcv_stream_kernel<3, 2, 1, false, (1 << ARC_U8)>;
}

#if defined(ARCV_TRACE) && ARCV_TRACE
ARCV_DEFINE_TRACE_COPY(k1_trace_copy_u8)
#endif

}  // namespace arcv
