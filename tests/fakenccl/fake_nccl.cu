// fake_nccl.cu -- TEST INFRASTRUCTURE, not part of the product.
//
// A stand-in for the handful of NCCL entry points libarcverify's collective
// fallback path uses (csrc/arcv_shard.cu: GetUniqueId, CommInitRank,
// CommDestroy, AllGather, Broadcast, GroupStart/End, GetErrorString), so that
// path can run with SEVERAL ranks as processes sharing one GPU -- real NCCL
// refuses two ranks on one device, and this pool offers one GPU per job.
// Semantics follow NCCL's for what the library calls (uint8 data, in-order
// collectives, every rank calling the same sequence); the implementation is
// deliberately simple and host-synchronous: each rank owns a device staging
// buffer exported with CUDA IPC through a POSIX shared-memory rendezvous, and
// every collective is "sync the stream, copy into staging, host barrier, copy
// out of the peers' staging, host barrier".  Loaded by the library through
// ARCV_NCCL_LIB (tests/test_nccl_fake_gpu.py).
#include <cuda_runtime.h>
#include <fcntl.h>
#include <sched.h>
#include <sys/mman.h>
#include <unistd.h>

#include <atomic>
#include <cstdio>
#include <cstdlib>
#include <cstring>

extern "C" {

typedef enum { ncclSuccess = 0, ncclUnhandledCudaError = 1, ncclSystemError = 2, ncclInternalError = 3,
               ncclInvalidArgument = 4 } ncclResult_t;
typedef struct { char internal[128]; } ncclUniqueId;
typedef int ncclDataType_t;
struct FakeComm;
typedef FakeComm *ncclComm_t;
}

namespace {

constexpr int kMaxRanks = 64;
constexpr size_t kStage = 64ull << 20;  // per-rank staging (largest collective in the tests: 24 MiB)

struct Shared {
    std::atomic<unsigned long long> arrive;  // barrier arrivals (monotonic)
    int nranks;
    cudaIpcMemHandle_t h[kMaxRanks];
    std::atomic<int> published[kMaxRanks];
};

}  // namespace

struct FakeComm {
    int rank, nranks;
    Shared *sh;
    char name[128];
    void *stage;
    void *peer[kMaxRanks];
    unsigned long long gen;  // barriers passed by this rank
};

namespace {

void barrier(FakeComm *c) {
    const unsigned long long target = (unsigned long long)(++c->gen) * c->nranks;
    c->sh->arrive.fetch_add(1);
    while (c->sh->arrive.load() < target) sched_yield();
}

ncclResult_t cuda_ok(cudaError_t e) { return e == cudaSuccess ? ncclSuccess : ncclUnhandledCudaError; }

// cudaMemcpy device-to-device returns before the copy completes: every copy is
// followed by a device synchronise before the barrier that publishes it
ncclResult_t copy_sync(void *dst, const void *src, size_t n) {
    ncclResult_t r = cuda_ok(cudaMemcpy(dst, src, n, cudaMemcpyDeviceToDevice));
    return r ? r : cuda_ok(cudaDeviceSynchronize());
}

}  // namespace

extern "C" {

ncclResult_t ncclGetUniqueId(ncclUniqueId *id) {
    memset(id, 0, sizeof(*id));
    snprintf(id->internal, sizeof(id->internal), "/arcv_fakenccl_%d_%ld", (int)getpid(), (long)random());
    return ncclSuccess;
}

ncclResult_t ncclCommInitRank(ncclComm_t *comm, int nranks, ncclUniqueId id, int rank) {
    if (nranks < 1 || nranks > kMaxRanks || rank < 0 || rank >= nranks) return ncclInvalidArgument;
    FakeComm *c = new FakeComm();
    c->rank = rank;
    c->nranks = nranks;
    c->gen = 0;
    snprintf(c->name, sizeof(c->name), "%s", id.internal);
    const int fd = shm_open(c->name, O_CREAT | O_RDWR, 0600);
    if (fd < 0) return ncclSystemError;
    if (ftruncate(fd, sizeof(Shared)) != 0) return ncclSystemError;
    void *m = mmap(nullptr, sizeof(Shared), PROT_READ | PROT_WRITE, MAP_SHARED, fd, 0);
    close(fd);
    if (m == MAP_FAILED) return ncclSystemError;
    c->sh = static_cast<Shared *>(m);  // zero-filled by ftruncate: atomics start at 0
    if (cudaMalloc(&c->stage, kStage) != cudaSuccess) return ncclUnhandledCudaError;
    if (cudaIpcGetMemHandle(&c->sh->h[rank], c->stage) != cudaSuccess) return ncclUnhandledCudaError;
    c->sh->published[rank].store(1);
    for (int r = 0; r < nranks; ++r)
        while (c->sh->published[r].load() == 0) sched_yield();
    for (int r = 0; r < nranks; ++r) {
        if (r == rank) {
            c->peer[r] = c->stage;
            continue;
        }
        if (cudaIpcOpenMemHandle(&c->peer[r], c->sh->h[r], cudaIpcMemLazyEnablePeerAccess) != cudaSuccess)
            return ncclUnhandledCudaError;
    }
    barrier(c);
    *comm = c;
    return ncclSuccess;
}

ncclResult_t ncclCommDestroy(ncclComm_t c) {
    if (!c) return ncclInvalidArgument;
    barrier(c);
    for (int r = 0; r < c->nranks; ++r)
        if (r != c->rank && c->peer[r]) cudaIpcCloseMemHandle(c->peer[r]);
    cudaFree(c->stage);
    munmap(c->sh, sizeof(Shared));
    if (c->rank == 0) shm_unlink(c->name);
    delete c;
    return ncclSuccess;
}

ncclResult_t ncclAllGather(const void *send, void *recv, size_t count, ncclDataType_t type, ncclComm_t c,
                           cudaStream_t st) {
    if (type != 1 || count > kStage) return ncclInvalidArgument;  // ncclUint8 only (what the library uses)
    ncclResult_t r = cuda_ok(cudaStreamSynchronize(st));
    if (r) return r;
    if ((r = copy_sync(c->stage, send, count))) return r;
    barrier(c);
    for (int q = 0; q < c->nranks; ++q)
        if ((r = copy_sync(static_cast<char *>(recv) + (size_t)q * count, c->peer[q], count))) return r;
    barrier(c);
    return ncclSuccess;
}

ncclResult_t ncclBroadcast(const void *send, void *recv, size_t count, ncclDataType_t type, int root,
                           ncclComm_t c, cudaStream_t st) {
    if (type != 1 || count > kStage || root < 0 || root >= c->nranks) return ncclInvalidArgument;
    ncclResult_t r = cuda_ok(cudaStreamSynchronize(st));
    if (r) return r;
    if (c->rank == root && (r = copy_sync(c->stage, send, count))) return r;
    barrier(c);
    if ((r = copy_sync(recv, c->peer[root], count))) return r;
    barrier(c);
    return ncclSuccess;
}

ncclResult_t ncclGroupStart() { return ncclSuccess; }  // collectives run eagerly, in call order
ncclResult_t ncclGroupEnd() { return ncclSuccess; }

const char *ncclGetErrorString(ncclResult_t r) { return r == ncclSuccess ? "fake nccl: ok" : "fake nccl: error"; }

}  // extern "C"
