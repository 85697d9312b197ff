// Diagnostic: host-side cost of the CUDA runtime calls on the compare call path
// (cudaPointerGetAttributes per pointer kind, a kernel launch, an event record).
//   nvcc -gencode arch=compute_100a,code=sm_100a -O2 -o /tmp/host_api_cost host_api_cost.cu && /tmp/host_api_cost
#include <chrono>
#include <cstdio>
#include <cstdlib>
#include <cuda_runtime.h>

__global__ void empty_kernel() {}

template <typename F>
static double us_per(F f, int n = 20000) {
    for (int i = 0; i < 100; ++i) f();
    auto t0 = std::chrono::steady_clock::now();
    for (int i = 0; i < n; ++i) f();
    auto t1 = std::chrono::steady_clock::now();
    return std::chrono::duration<double, std::micro>(t1 - t0).count() / n;
}

int main() {
    void *d, *h;
    cudaMalloc(&d, 1 << 20);
    cudaMallocHost(&h, 1 << 20);
    void *pg = malloc(1 << 20);
    cudaPointerAttributes a;
    printf("cudaPointerGetAttributes device  %.3f us\n", us_per([&] { cudaPointerGetAttributes(&a, d); }));
    printf("cudaPointerGetAttributes pinned  %.3f us\n", us_per([&] { cudaPointerGetAttributes(&a, h); }));
    printf("cudaPointerGetAttributes pageable %.3f us\n", us_per([&] { cudaPointerGetAttributes(&a, pg); }));
    cudaStream_t s;
    cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking);
    cudaEvent_t e;
    cudaEventCreate(&e);
    printf("cudaEventRecord                  %.3f us\n", us_per([&] { cudaEventRecord(e, s); }));
    printf("empty kernel launch              %.3f us\n", us_per([&] { empty_kernel<<<1, 32, 0, s>>>(); }));
    cudaStreamSynchronize(s);
    printf("launch + stream sync             %.3f us\n", us_per([&] { empty_kernel<<<1, 32, 0, s>>>(); cudaStreamSynchronize(s); }, 2000));
    return 0;
}
