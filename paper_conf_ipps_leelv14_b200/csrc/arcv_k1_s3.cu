// arcv_k1_s3.cu -- K1 (arcv_stream_kernel) with 3 pipeline stages, min 2 CTAs
// per SM; one translation unit per stage count (arcv_kernels.h).
#include <cuda_runtime.h>


#include "arcv_device.cuh"
#include "arcv_kernels.h"

namespace arcv {

KernelFnN<1> k1_s3_1() { return arcv_stream_kernel<3, 2, 1>; }
KernelFnN<kMaxInlineSegs> k1_s3_n() { return arcv_stream_kernel<3, 2, kMaxInlineSegs>; }
KernelFnN<1> k1_s3_1x() { return arcv_stream_kernel<3, 2, 1, true>; }  // sharded: exchange fused

// K2: the separate report kernel (used with S = 2 K1s or ARCV_FUSED=0)
KernelFnN<1> k2_fn_1() { return arcv_compact_kernel<1>; }
KernelFnN<kMaxInlineSegs> k2_fn_n() { return arcv_compact_kernel<kMaxInlineSegs>; }

// The trace buffer is a __device__ variable of each module (translation unit):
// this one holds the generic K1s and K2, the dtype-specialised K1s have their own.
ARCV_DEFINE_TRACE_COPY(k1_trace_copy)

}  // namespace arcv
