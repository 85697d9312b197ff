// arcv_k1_s2.cu -- K1 (arcv_stream_kernel) with 2 pipeline stages, min 3 CTAs
// per SM; one translation unit per stage count (arcv_kernels.h).
#include <cuda_runtime.h>

#include <vector>

#include "arcv_device.cuh"
#include "arcv_kernels.h"

namespace arcv {

KernelFnN<1> k1_s2_1() { return arcv_stream_kernel<2, 3, 1>; }
KernelFnN<kMaxInlineSegs> k1_s2_n() { return arcv_stream_kernel<2, 3, kMaxInlineSegs>; }
KernelFnN<1> k1_s2_1x() { return arcv_stream_kernel<2, 3, 1, true>; }  // sharded: exchange fused

}  // namespace arcv
