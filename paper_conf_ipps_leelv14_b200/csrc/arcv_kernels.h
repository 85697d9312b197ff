// arcv_kernels.h -- host-side handles of the compare kernels.  K1
// (arcv_stream_kernel<S, MINB, NSEG>) is instantiated once per stage count in
// its own translation unit (arcv_k1_s<S>.cu) so the variants compile in
// parallel; K2 (arcv_compact_kernel<NSEG>) lives with the default K1 (S = 3).
// Each TU exports plain functions returning the kernel's host-stub address,
// which is what cudaLaunchKernelEx / cudaFuncSetAttribute take.
#pragma once
#include "arcv_types.h"

namespace arcv {

template <int NSEG>
using KernelFnN = void (*)(ParamsN<NSEG>);

// K1 with S stages (S in {2, 3, 4, 6}); `xf`: the variant with the sharded
// exchange fused into its tail (single-segment parameter blocks only).
KernelFnN<1> k1_fn_1(int stages, bool xf = false);
KernelFnN<kMaxInlineSegs> k1_fn_n(int stages);
// per-TU providers (arcv_k1_s<S>.cu)
#define ARCV_K1_DECL(S)                    \
    KernelFnN<1> k1_s##S##_1();            \
    KernelFnN<1> k1_s##S##_1x();           \
    KernelFnN<kMaxInlineSegs> k1_s##S##_n();
ARCV_K1_DECL(2)
ARCV_K1_DECL(3)
ARCV_K1_DECL(4)
ARCV_K1_DECL(6)
#undef ARCV_K1_DECL
// K1 with 3 stages specialised for one dtype (single-region calls; `xf` as
// above), one translation unit per dtype (arcv_k1_s3_dt<dtype>.cu)
KernelFnN<1> k1_s3_1_f32(bool xf);
KernelFnN<1> k1_s3_1_f64(bool xf);
KernelFnN<1> k1_s3_1_i32(bool xf);
KernelFnN<1> k1_s3_1_i64(bool xf);
KernelFnN<1> k1_s3_1_u8(bool xf);
KernelFnN<1> k1_fn_1_dt(int stages, bool xf, int dtype);  // nullptr: no specialisation
// K1 with 3 stages for batches of fp32 / fp64 / int32 regions (arcv_k1_s3_dtbatch.cu)
KernelFnN<kMaxInlineSegs> k1_s3_n_fi();
// K2 (arcv_k1_s3.cu)
KernelFnN<1> k2_fn_1();
KernelFnN<kMaxInlineSegs> k2_fn_n();
// ARCV_TRACE builds: copy (and clear) the phase stamps the kernels wrote
int k1_trace_copy(unsigned long long *out, size_t bytes);
int k1_trace_copy_f32(unsigned long long *out, size_t bytes);
int k1_trace_copy_f64(unsigned long long *out, size_t bytes);
int k1_trace_copy_i32(unsigned long long *out, size_t bytes);
int k1_trace_copy_i64(unsigned long long *out, size_t bytes);
int k1_trace_copy_u8(unsigned long long *out, size_t bytes);
int k1_trace_copy_batch(unsigned long long *out, size_t bytes);

}  // namespace arcv
