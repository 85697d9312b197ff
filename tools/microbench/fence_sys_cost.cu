// Diagnostic: what a fence.acq_rel.sys costs at the end of a kernel that wrote
// N 24-byte entries into mapped pinned host memory (the direct report route),
// measured as the kernel's event time from an idle stream, with and without
// the fence before the final flag store.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O2 -o /tmp/fence fence_sys_cost.cu && /tmp/fence
#include <cstdio>
#include <cuda_runtime.h>

__global__ void k(unsigned long long *host, int n_entries, int fenced, unsigned long long seq) {
    // entries spread over the grid like the report phase (one thread per word)
    for (int w = blockIdx.x * blockDim.x + threadIdx.x; w < 3 * n_entries; w += gridDim.x * blockDim.x)
        host[8 + w] = seq + w;
    __syncthreads();
    if (threadIdx.x == 0) {
        asm volatile("fence.acq_rel.gpu;" ::: "memory");
        unsigned long long prev = atomicAdd(host ? (unsigned long long *)nullptr + 0 : nullptr, 0ull);
        (void)prev;
    }
}

__global__ void k2(unsigned long long *host, unsigned long long *ctr, int n_entries, int fenced,
                   unsigned long long seq, unsigned long long base) {
    for (int w = blockIdx.x * blockDim.x + threadIdx.x; w < 3 * n_entries; w += gridDim.x * blockDim.x)
        host[8 + w] = seq + w;
    __syncthreads();
    __shared__ int last;
    if (threadIdx.x == 0) {
        asm volatile("fence.acq_rel.gpu;" ::: "memory");
        last = (atomicAdd(ctr, 1ull) - base) == gridDim.x - 1;
    }
    __syncthreads();
    if (last && threadIdx.x == 0) {
        if (fenced) asm volatile("fence.acq_rel.sys;" ::: "memory");
        *(volatile unsigned long long *)host = seq;
    }
}

int main() {
    unsigned long long *h, *d, *ctr;
    cudaHostAlloc(&h, 64 << 20, cudaHostAllocMapped);
    cudaHostGetDevicePointer((void **)&d, h, 0);
    cudaMalloc(&ctr, 8);
    cudaMemset(ctr, 0, 8);
    cudaStream_t s;
    cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking);
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    unsigned long long seq = 1, base = 0;
    const int grid = 296;
    for (int n : {0, 516, 4096, 8190}) {
        for (int fenced = 0; fenced < 2; ++fenced) {
            double tot = 0;
            const int reps = 500;
            for (int i = 0; i < reps + 20; ++i) {
                cudaStreamSynchronize(s);
                cudaEventRecord(e0, s);
                k2<<<grid, 256, 0, s>>>(d, ctr, n, fenced, ++seq, base);
                base += grid;
                cudaEventRecord(e1, s);
                cudaEventSynchronize(e1);
                float ms;
                cudaEventElapsedTime(&ms, e0, e1);
                if (i >= 20) tot += ms * 1e3;
            }
            printf("entries %5d  %-9s: %.2f us per kernel (events, idle stream)\n", n, fenced ? "fence.sys" : "no fence",
                   tot / reps);
        }
    }
    printf("err %s\n", cudaGetErrorString(cudaGetLastError()));
    return 0;
}
