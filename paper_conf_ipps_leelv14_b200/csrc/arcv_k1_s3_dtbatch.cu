// arcv_k1_s3_dtbatch.cu -- K1 with 3 stages, min 2 CTAs per SM, for batches of
// fp32 / fp64 / int32 regions only (kDtmFloatI32: the twelve-benchmark batch C3
// and most region lists); arcv_kernels.h.
#include <cuda_runtime.h>

#include "arcv_device.cuh"
#include "arcv_kernels.h"

namespace arcv {

KernelFnN<kMaxInlineSegs> k1_s3_n_fi() { return arcv_stream_kernel<3, 2, kMaxInlineSegs, false, kDtmFloatI32>; }

#if defined(ARCV_TRACE) && ARCV_TRACE
ARCV_DEFINE_TRACE_COPY(k1_trace_copy_batch)
#endif

}  // namespace arcv
