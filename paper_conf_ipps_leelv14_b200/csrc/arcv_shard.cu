// arcv_shard.cu -- sharding one large region across the GPUs of one box
// (DESIGN.md sec. 2 step a8).
//
// The paper verifies on one GPU.  Here each rank compares its
// contiguous shard locally (a2-a5), then ONE ncclAllGather exchanges fixed-size
// packets {32-byte header, first K local mismatches}; a merge kernel on every
// rank turns the gathered headers into the merge plan (global index offset,
// report position and contribution per rank) and writes the global report in
// rank order = index order.  Entries that do not fit in a packet (a rank whose
// contribution exceeds K) follow in one grouped ncclBroadcast per contributing
// rank.  NCCL is opened at run time (dlopen of libnccl.so.2 -- the copy torch
// already loaded, if any), so the library loads on machines without NCCL.
#include <cuda_runtime.h>
#include <dlfcn.h>
#include <nccl.h>

#include <algorithm>
#include <cstring>
#include <vector>

#include "arc_verify.h"
#include "arcv_internal.h"
#include "arcv_merge.h"

namespace arcv {

constexpr uint64_t kPacketEntries = 4096;  // K: entries carried in the all-gather

// Every block rebuilds the plan in shared memory (p <= 256 headers), then the
// grid copies the packet entries that belong to the global report, adding each
// rank's index offset.  Block 0 publishes [global header, per-rank headers].
__global__ void __launch_bounds__(256) arcv_merge_kernel(const uint8_t *gathered, int p, uint64_t stride,
                                                         uint64_t K, uint64_t max_report, arc_mismatch_t *dst,
                                                         arc_shard_header_t *hdr_out) {
    __shared__ arc_shard_header_t hdr[kMaxRanks];
    __shared__ arc_shard_plan_t plan[kMaxRanks];
    __shared__ uint64_t cum[kMaxRanks + 1];
    __shared__ arc_shard_header_t glob;
    for (int r = threadIdx.x; r < p; r += blockDim.x)
        hdr[r] = *reinterpret_cast<const arc_shard_header_t *>(gathered + (uint64_t)r * stride);
    __syncthreads();
    if (threadIdx.x == 0) {
        merge_plan_impl(hdr, p, max_report, plan, &glob);
        cum[0] = 0;
        for (int r = 0; r < p; ++r) cum[r + 1] = cum[r] + (plan[r].contrib < K ? plan[r].contrib : K);
        if (blockIdx.x == 0) {
            hdr_out[0] = glob;
            for (int r = 0; r < p; ++r) hdr_out[1 + r] = hdr[r];
        }
    }
    __syncthreads();
    const uint64_t total = cum[p];
    for (uint64_t gi = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; gi < total;
         gi += (uint64_t)gridDim.x * blockDim.x) {
        int r = 0;
        while (cum[r + 1] <= gi) ++r;
        const uint64_t j = gi - cum[r];
        const arc_mismatch_t *src =
            reinterpret_cast<const arc_mismatch_t *>(gathered + (uint64_t)r * stride + sizeof(arc_shard_header_t)) + j;
        arc_mismatch_t e = *src;
        e.index += plan[r].index_offset;
        dst[plan[r].prefix + j] = e;
    }
}

__global__ void arcv_offset_kernel(arc_mismatch_t *e, uint64_t count, uint64_t off) {
    for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < count; i += (uint64_t)gridDim.x * blockDim.x)
        e[i].index += off;
}

// ------------------------------------------------------------------- NCCL
struct NcclApi {
    void *h = nullptr;
    ncclResult_t (*GetUniqueId)(ncclUniqueId *) = nullptr;
    ncclResult_t (*CommInitRank)(ncclComm_t *, int, ncclUniqueId, int) = nullptr;
    ncclResult_t (*CommDestroy)(ncclComm_t) = nullptr;
    ncclResult_t (*AllGather)(const void *, void *, size_t, ncclDataType_t, ncclComm_t, cudaStream_t) = nullptr;
    ncclResult_t (*Broadcast)(const void *, void *, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t) = nullptr;
    ncclResult_t (*GroupStart)() = nullptr;
    ncclResult_t (*GroupEnd)() = nullptr;
    const char *(*GetErrorString)(ncclResult_t) = nullptr;
};
static NcclApi nccl;

static int load_nccl() {
    if (nccl.h) return ARC_OK;
    // ARCV_NCCL_LIB (diagnostics / tests) names the library explicitly and wins;
    // otherwise the copy torch already loaded, else the system's.
    const char *env = getenv("ARCV_NCCL_LIB");
    void *h = (env && *env) ? dlopen(env, RTLD_NOW | RTLD_LOCAL) : dlopen("libnccl.so.2", RTLD_NOW | RTLD_NOLOAD);
    if (!h && !(env && *env)) h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
    if (!h) {
        set_error("cannot load NCCL: %s", dlerror());
        return ARC_E_NCCL;
    }
#define LOAD(field, sym)                                                   \
    *reinterpret_cast<void **>(&nccl.field) = dlsym(h, sym);               \
    if (!nccl.field) {                                                     \
        set_error("NCCL symbol %s missing", sym);                          \
        return ARC_E_NCCL;                                                 \
    }
    LOAD(GetUniqueId, "ncclGetUniqueId");
    LOAD(CommInitRank, "ncclCommInitRank");
    LOAD(CommDestroy, "ncclCommDestroy");
    LOAD(AllGather, "ncclAllGather");
    LOAD(Broadcast, "ncclBroadcast");
    LOAD(GroupStart, "ncclGroupStart");
    LOAD(GroupEnd, "ncclGroupEnd");
    LOAD(GetErrorString, "ncclGetErrorString");
#undef LOAD
    nccl.h = h;
    return ARC_OK;
}

static int nccl_fail(ncclResult_t r, const char *what) {
    set_error("%s: %s", what, nccl.GetErrorString ? nccl.GetErrorString(r) : "?");
    return ARC_E_NCCL;
}
#define NK(call)                                                  \
    do {                                                          \
        ncclResult_t r_ = (call);                                 \
        if (r_ != ncclSuccess) return nccl_fail(r_, #call);       \
    } while (0)
#define CK(call)                                                  \
    do {                                                          \
        cudaError_t e_ = (call);                                  \
        if (e_ != cudaSuccess) return cuda_fail(e_, #call);       \
    } while (0)

int shard_init(Ctx &c, const void *id) {
    int st = load_nccl();
    if (st) return st;
    if (c.nranks > kMaxRanks) {
        set_error("nranks %d > %d", c.nranks, kMaxRanks);
        return ARC_E_UNSUPPORTED;
    }
    ncclUniqueId uid;
    memcpy(&uid, id, sizeof(uid));
    ncclComm_t comm;
    NK(nccl.CommInitRank(&comm, c.nranks, uid, c.rank));
    c.nccl_comm = comm;
    return ARC_OK;
}

void shard_finalize(Ctx &c) {
    if (c.nccl_comm && nccl.CommDestroy) nccl.CommDestroy(static_cast<ncclComm_t>(c.nccl_comm));
    c.nccl_comm = nullptr;
    if (c.merge_dev) cudaFree(c.merge_dev);
    c.merge_dev = nullptr;
}

static int grow_bytes(uint8_t **p, size_t *cap, size_t need, cudaStream_t st) {
    if (need <= *cap) return ARC_OK;
    if (*p) {
        CK(cudaStreamSynchronize(st));
        CK(cudaFree(*p));
    }
    *p = nullptr;
    *cap = 0;
    const size_t ncap = std::max(need, (size_t)4096);
    cudaError_t e = cudaMalloc(reinterpret_cast<void **>(p), ncap);
    if (e != cudaSuccess) {
        cudaGetLastError();
        set_error("cudaMalloc(%zu) failed", ncap);
        return ARC_E_NOMEM;
    }
    *cap = ncap;
    return ARC_OK;
}

static int ensure_hdr_buffers(Ctx &c, int p) {
    if (!c.merge_dev) {
        cudaError_t e = cudaMalloc(&c.merge_dev, (kMaxRanks + 1) * sizeof(arc_shard_header_t));
        if (e != cudaSuccess) {
            cudaGetLastError();
            set_error("cudaMalloc(merge headers)");
            return ARC_E_NOMEM;
        }
    }
    if (c.hdr_host_cap < (size_t)(p + 1)) {
        if (c.hdr_host) CK(cudaFreeHost(c.hdr_host));
        c.hdr_host = nullptr;
        c.hdr_host_cap = 0;
        CK(cudaMallocHost(&c.hdr_host, (kMaxRanks + 1) * sizeof(arc_shard_header_t)));
        c.hdr_host_cap = kMaxRanks + 1;
    }
    return ARC_OK;
}

// Local compare of one shard into a packet (header + local entries).
static int local_packet(Ctx &c, const arc_verify_region_t &r, uint8_t *packet) {
    arc_mismatch_t *entries = reinterpret_cast<arc_mismatch_t *>(packet + sizeof(arc_shard_header_t));
    arc_verify_result_t res;
    memset(&res, 0, sizeof(res));
    res.report = entries;  // only checked for non-NULL; the kernel writes via dev_reports
    Acc a;
    int st = run_local(c, &r, 1, &res, &entries, false, &a);
    if (st) return st;
    int hs = ensure_hdr_buffers(c, 1);
    if (hs) return hs;
    arc_shard_header_t h{r.n, a.count, a.max_abs_bits, a.max_rel_bits};
    c.hdr_host[0] = h;
    CK(cudaMemcpyAsync(packet, c.hdr_host, sizeof(h), cudaMemcpyHostToDevice, c.stream));
    CK(cudaStreamSynchronize(c.stream));  // hdr_host is reused
    return ARC_OK;
}

// Merge gathered packets on the device; leaves per-rank headers + global header
// in c.hdr_host[0..p] and the plan in `plan`.  `dst` = device report target.
static int merge_gathered(Ctx &c, const uint8_t *gathered, int p, uint64_t K, uint64_t max_report,
                          arc_mismatch_t *dst, std::vector<arc_shard_plan_t> &plan) {
    int st = ensure_hdr_buffers(c, p);
    if (st) return st;
    const uint64_t stride = arc_verify_packet_bytes(K);
    const int grid = std::max(1, std::min(c.num_sms, (int)((std::min(K, max_report) * p + 255) / 256)));
    arcv_merge_kernel<<<grid, 256, 0, c.stream>>>(gathered, p, stride, K, max_report, dst, c.merge_dev);
    CK(cudaGetLastError());
    c.launches++;
    CK(cudaMemcpyAsync(c.hdr_host, c.merge_dev, (p + 1) * sizeof(arc_shard_header_t), cudaMemcpyDeviceToHost,
                       c.stream));
    CK(cudaStreamSynchronize(c.stream));
    plan.resize(p);
    arc_shard_header_t g;
    merge_plan_impl(c.hdr_host + 1, p, max_report, plan.data(), &g);
    return ARC_OK;
}

void fill_result(const arc_shard_header_t &g, uint64_t max_report, arc_verify_result_t *res) {
    res->n = g.n;
    res->n_mismatch = g.n_mismatch;
    memcpy(&res->max_abs_err, &g.max_abs_bits, 8);
    memcpy(&res->max_rel_err, &g.max_rel_bits, 8);
    res->n_reported = std::min(g.n_mismatch, max_report);
}

// Device target for the global report (caller's device buffer, or staging).
int report_target(Ctx &c, arc_verify_result_t *result, uint64_t cap, arc_mismatch_t **dst, bool *host) {
    *dst = nullptr;
    *host = false;
    if (cap == 0) return ARC_OK;
    if (classify(result->report, c.device) == PK_DEVICE) {
        *dst = result->report;
        return ARC_OK;
    }
    if (c.report_stage_cap < cap) {
        if (c.report_stage) {
            CK(cudaStreamSynchronize(c.stream));
            CK(cudaFree(c.report_stage));
        }
        c.report_stage = nullptr;
        c.report_stage_cap = 0;
        cudaError_t e = cudaMalloc(&c.report_stage, cap * sizeof(arc_mismatch_t));
        if (e != cudaSuccess) {
            cudaGetLastError();
            set_error("cudaMalloc(report staging)");
            return ARC_E_NOMEM;
        }
        c.report_stage_cap = cap;
    }
    *dst = c.report_stage;
    *host = true;
    return ARC_OK;
}

int shard_compare(Ctx &c, const arc_verify_region_t &r, arc_verify_result_t *result) {
    // the device-driven peer-memory exchange (arcv_peer.cu) when the windows are
    // open and large enough -- uniform across ranks (same max_report, same cap)
    if (c.peer_ready && r.max_report <= c.win_cap) return peer_compare(c, r, result);
    if (!c.nccl_comm) {
        set_error(c.peer_ready ? "max_report %llu exceeds the peer window capacity and no NCCL communicator"
                               : "sharded mode needs arc_verify_peer_open or an NCCL id (max_report %llu)",
                  (unsigned long long)r.max_report);
        return ARC_E_UNSUPPORTED;
    }
    int st = validate_region(r.out, r.ref, r.n, r.dtype, r.abs_tol, r.rel_tol, r.max_report, result);
    if (st) return st;
    const int p = c.nranks;
    const uint64_t K = std::min<uint64_t>(r.max_report, kPacketEntries);
    const uint64_t local_cap = std::min<uint64_t>(r.max_report, r.n);
    st = grow_bytes(&c.packet, &c.packet_cap, arc_verify_packet_bytes(std::max(K, local_cap)), c.stream);
    if (st) return st;
    st = grow_bytes(&c.gathered, &c.gathered_cap, (size_t)p * arc_verify_packet_bytes(K), c.stream);
    if (st) return st;
    st = local_packet(c, r, c.packet);
    if (st) return st;
    ncclComm_t comm = static_cast<ncclComm_t>(c.nccl_comm);
    NK(nccl.AllGather(c.packet, c.gathered, arc_verify_packet_bytes(K), ncclUint8, comm, c.stream));
    // global report capacity: all ranks agree on the global count only after the
    // merge, so size the target by the caller's capacity contract.
    arc_mismatch_t *dst;
    bool host_report;
    st = report_target(c, result, r.max_report, &dst, &host_report);
    if (st) return st;
    std::vector<arc_shard_plan_t> plan;
    st = merge_gathered(c, c.gathered, p, K, r.max_report, dst, plan);
    if (st) return st;
    const arc_shard_header_t g = c.hdr_host[0];
    // phase B: contributions larger than a packet
    bool any = false;
    for (int q = 0; q < p; ++q) any |= plan[q].contrib > K;
    if (any) {
        NK(nccl.GroupStart());
        for (int q = 0; q < p; ++q) {
            if (plan[q].contrib <= K) continue;
            const size_t bytes = (plan[q].contrib - K) * sizeof(arc_mismatch_t);
            const void *src = c.packet + sizeof(arc_shard_header_t) + K * sizeof(arc_mismatch_t);
            NK(nccl.Broadcast(src, dst + plan[q].prefix + K, bytes, ncclUint8, q, comm, c.stream));
        }
        NK(nccl.GroupEnd());
        for (int q = 0; q < p; ++q) {
            if (plan[q].contrib <= K) continue;
            const uint64_t cnt = plan[q].contrib - K;
            const int blocks = (int)std::min<uint64_t>((cnt + 255) / 256, (uint64_t)c.num_sms * 4);
            arcv_offset_kernel<<<blocks, 256, 0, c.stream>>>(dst + plan[q].prefix + K, cnt, plan[q].index_offset);
            CK(cudaGetLastError());
            c.launches++;
        }
    }
    fill_result(g, r.max_report, result);
    if (host_report && result->n_reported)
        CK(cudaMemcpyAsync(result->report, dst, result->n_reported * sizeof(arc_mismatch_t), cudaMemcpyDeviceToHost,
                           c.stream));
    CK(cudaStreamSynchronize(c.stream));
    return ARC_OK;
}

}  // namespace arcv

using namespace arcv;

extern "C" {

size_t arc_verify_packet_bytes(uint64_t entries) {
    return sizeof(arc_shard_header_t) + (size_t)entries * sizeof(arc_mismatch_t);
}

int arc_verify_merge_plan(const arc_shard_header_t *hdrs, int nranks, uint64_t max_report, arc_shard_plan_t *plan,
                          arc_shard_header_t *global) {
    if (!hdrs || !plan || !global || nranks < 1) {
        set_error("merge_plan: bad arguments");
        return ARC_E_INVAL;
    }
    merge_plan_impl(hdrs, nranks, max_report, plan, global);
    return ARC_OK;
}

int arc_verify_get_unique_id(void *id) {
    if (!id) return ARC_E_INVAL;
    int st = load_nccl();
    if (st) return st;
    ncclUniqueId uid;
    NK(nccl.GetUniqueId(&uid));
    memcpy(id, &uid, sizeof(uid));
    return ARC_OK;
}

int arc_verify_shard_local(const void *out, const void *ref, uint64_t n, arc_dtype_t dtype, double abs_tol,
                           double rel_tol, uint64_t max_report, void *packet_dev, uint64_t packet_entries) {
    if (!g_ctx) return ARC_E_NOINIT;
    // the local report holds min(max_report, n) entries: it must fit the packet
    if (std::min<uint64_t>(max_report, n) > packet_entries) {
        set_error("shard_local: min(max_report, n) = %llu entries exceed the packet capacity %llu",
                  (unsigned long long)std::min<uint64_t>(max_report, n), (unsigned long long)packet_entries);
        return ARC_E_INVAL;
    }
    if (!packet_dev || classify(packet_dev, g_ctx->device) != PK_DEVICE) {
        set_error("packet must be device memory on the library's device");
        return ARC_E_INVAL;
    }
    arc_verify_region_t r{out, ref, n, dtype, abs_tol, rel_tol, max_report, nullptr, nullptr};
    return local_packet(*g_ctx, r, static_cast<uint8_t *>(packet_dev));
}

int arc_verify_shard_merge(const void *gathered_dev, int nranks, uint64_t packet_entries, uint64_t max_report,
                           arc_verify_result_t *result) {
    if (!g_ctx) return ARC_E_NOINIT;
    Ctx &c = *g_ctx;
    if (!gathered_dev || nranks < 1 || nranks > kMaxRanks || !result || (max_report > 0 && !result->report)) {
        set_error("shard_merge: bad arguments");
        return ARC_E_INVAL;
    }
    arc_mismatch_t *dst;
    bool host_report;
    int st = report_target(c, result, max_report, &dst, &host_report);
    if (st) return st;
    std::vector<arc_shard_plan_t> plan;
    st = merge_gathered(c, static_cast<const uint8_t *>(gathered_dev), nranks, packet_entries, max_report, dst, plan);
    if (st) return st;
    for (int q = 0; q < nranks; ++q)
        if (plan[q].contrib > packet_entries) {
            set_error("rank %d contributes %llu entries > packet capacity %llu", q,
                      (unsigned long long)plan[q].contrib, (unsigned long long)packet_entries);
            return ARC_E_UNSUPPORTED;
        }
    fill_result(c.hdr_host[0], max_report, result);
    if (host_report && result->n_reported) {
        CK(cudaMemcpyAsync(result->report, dst, result->n_reported * sizeof(arc_mismatch_t), cudaMemcpyDeviceToHost,
                           c.stream));
        CK(cudaStreamSynchronize(c.stream));
    }
    return ARC_OK;
}

}  // extern "C"
