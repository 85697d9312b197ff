// Diagnostic: device-side cost (CUDA events around the launch, idle stream
// before each launch -- how a compare call is timed) and host-side API time of
// a normal vs a cooperative launch of the same kernel shape as K1 (296 CTAs x
// 288 threads, 96 KB dynamic shared memory).
//   nvcc -gencode arch=compute_100a,code=sm_100a -O2 -o /tmp/coop coop_launch_cost.cu && /tmp/coop
#include <chrono>
#include <cstdio>
#include <cuda_runtime.h>

__global__ void k(int *x) {
    extern __shared__ int sm[];
    if (threadIdx.x == 0 && blockIdx.x == 0 && x) sm[0] = *x;
}

int main() {
    cudaStream_t s;
    cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking);
    const size_t smem = 98496;
    cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    int sms = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    for (int coop = 0; coop < 2; ++coop) {
        for (int pass = 0; pass < 2; ++pass) {
            double dev = 0, host = 0;
            const int n = 2000;
            for (int i = 0; i < n; ++i) {
                cudaStreamSynchronize(s);
                cudaEventRecord(e0, s);
                cudaLaunchConfig_t cfg = {};
                cfg.gridDim = dim3(2 * sms);
                cfg.blockDim = dim3(288);
                cfg.dynamicSmemBytes = smem;
                cfg.stream = s;
                cudaLaunchAttribute at[1];
                at[0].id = cudaLaunchAttributeCooperative;
                at[0].val.cooperative = 1;
                cfg.attrs = at;
                cfg.numAttrs = coop;
                auto t0 = std::chrono::steady_clock::now();
                cudaLaunchKernelEx(&cfg, k, (int *)nullptr);
                auto t1 = std::chrono::steady_clock::now();
                cudaEventRecord(e1, s);
                cudaEventSynchronize(e1);
                float ms;
                cudaEventElapsedTime(&ms, e0, e1);
                dev += ms * 1e3;
                host += std::chrono::duration<double, std::micro>(t1 - t0).count();
            }
            if (pass) printf("%s launch: device (events, idle stream) %.2f us, host API %.2f us\n",
                             coop ? "cooperative" : "normal     ", dev / n, host / n);
        }
    }
    printf("err %s\n", cudaGetErrorString(cudaGetLastError()));
    return 0;
}
