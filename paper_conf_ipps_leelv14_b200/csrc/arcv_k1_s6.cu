// arcv_k1_s6.cu -- K1 (arcv_stream_kernel) with 6 pipeline stages, min 1 CTAs
// per SM; one translation unit per stage count (arcv_kernels.h).
#include <cuda_runtime.h>

#include <vector>

#include "arcv_device.cuh"
#include "arcv_kernels.h"

namespace arcv {

KernelFnN<1> k1_s6_1() { return arcv_stream_kernel<6, 1, 1>; }
KernelFnN<kMaxInlineSegs> k1_s6_n() { return arcv_stream_kernel<6, 1, kMaxInlineSegs>; }
KernelFnN<1> k1_s6_1x() { return arcv_stream_kernel<6, 1, 1, true>; }  // sharded: exchange fused

}  // namespace arcv
