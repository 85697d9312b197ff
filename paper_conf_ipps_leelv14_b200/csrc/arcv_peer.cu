// arcv_peer.cu -- the cross-GPU exchange of a sharded comparison over peer
// memory (NVLink 5 / NVSwitch P2P), fused into one kernel (
// SURVEY.md sec. 8(a) step a8 and 8(e)).
//
// The paper verifies on one GPU; sharding one large output array across
// the GPUs of a box is this build's extension (reading R-shard).  The exchange
// the merge needs is tiny -- a 32-byte header per rank plus the first
// max_report mismatches -- so its cost is latency, not bandwidth.  Instead of
// host-driven NCCL calls (several host round trips per compare), every rank
// owns a symmetric "window" in its HBM, mapped into every other rank with CUDA
// IPC, and one kernel per call does the whole exchange on the device:
//
//   K1 (arcv_device.cuh) writes the rank's local report straight into its own
//   window (packet[parity]) and the local summary into a device mirror;
//   arcv_peer_kernel then
//     1. publishes: block 0 writes the local header into its window, fences at
//        system scope, and stores the call's sequence number into flag slot
//        [parity][rank] of EVERY rank's window (st.release.sys over NVLink);
//     2. waits: thread 0 of every block spins (ld.acquire.sys) until all p flags
//        of its own window carry the sequence number;
//     3. merges: every block reads the p headers from the peers' windows (P2P
//        loads), rebuilds the merge plan (arcv_merge.h, the one definition), and
//        the grid copies each rank's contributing entries from that rank's
//        window into the global report, adding the rank's index offset;
//     4. completes: the last block writes the global header to mapped host
//        memory and then the call's completion word, which the host polls.
//   One host wake-up per call; no NCCL call on the path.
//
// Reuse safety (double buffering by call parity): a rank overwrites
// packet[par] / flag[par][*] again only at call s + 2, which needs every peer's
// flag of call s + 1, which every peer publishes only after its merge of call s
// has finished (same stream).  Flags hold the sequence number itself, so a
// stale flag (s - 2) never satisfies a wait for s.
//
// The wait is bounded (a %globaltimer deadline): a peer that never arrives
// yields ARC_E_CUDA ("peer exchange timed out") instead of a hung GPU.
#include <cuda_runtime.h>

#include <algorithm>
#include <cstring>

#include "arc_verify.h"
#include "arcv_internal.h"

namespace arcv {

constexpr size_t kFlagBytes = 2 * kMaxRanks * sizeof(unsigned long long);  // [2 parities][kMaxRanks]
constexpr unsigned long long kPeerTimeoutNs = 60ull * 1000 * 1000 * 1000;  // 60 s

__host__ __device__ inline size_t packet_stride(uint64_t cap) {
    return (sizeof(arc_shard_header_t) + (size_t)cap * sizeof(arc_mismatch_t) + 127) & ~(size_t)127;
}
__host__ __device__ inline unsigned long long *flag_slot(uint8_t *win, int par, int r) {
    return reinterpret_cast<unsigned long long *>(win) + (size_t)par * kMaxRanks + r;
}
__host__ __device__ inline uint8_t *packet_at(uint8_t *win, uint64_t cap, int par) {
    return win + kFlagBytes + (size_t)par * packet_stride(cap);
}

struct PeerParams {
    uint8_t *const *win;            // [p] window base pointers (own + IPC-mapped peers)
    int rank, p, par;
    unsigned long long s;           // collective sequence number = flag value
    uint64_t n_local, max_report, cap;
    const Acc *mirror;              // local summary (written by the local compare)
    arc_mismatch_t *dst;            // global report target (device memory or HBM staging), or nullptr
    arc_mismatch_t *dst_alias;      // device alias of the caller's pinned host report, or nullptr:
                                    // used instead of dst when the global report has <= kDirectDyn
                                    // entries (the host then skips its D2H copy; same rule there)
    arc_shard_header_t *out;        // mapped host: [0] global header, [1].n = status (1 = timeout)
    unsigned long long *done;       // monotonic finished-block counter
    unsigned long long done_base;
    unsigned long long *done_flag;  // mapped completion word
    unsigned long long seq;
};

__device__ __forceinline__ void st_release_sys(unsigned long long *p, unsigned long long v) {
    asm volatile("st.release.sys.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ unsigned long long ld_acquire_sys(const unsigned long long *p) {
    unsigned long long v;
    asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
// message-passing fences (no fence.sc needed; see arcv_device.cuh fence_gpu/fence_sys)
__device__ __forceinline__ void peer_fence_gpu() { asm volatile("fence.acq_rel.gpu;" ::: "memory"); }
__device__ __forceinline__ void peer_fence_sys() { asm volatile("fence.acq_rel.sys;" ::: "memory"); }
__device__ __forceinline__ unsigned long long ld_volatile(const unsigned long long *p) {
    return *reinterpret_cast<const volatile unsigned long long *>(p);
}
__device__ __forceinline__ unsigned long long globaltimer() {
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
}

__global__ void __launch_bounds__(256) arcv_peer_kernel(const __grid_constant__ PeerParams q) {
    __shared__ arc_shard_header_t hdr[kMaxRanks];
    __shared__ arc_shard_plan_t plan[kMaxRanks];
    __shared__ uint64_t cum[kMaxRanks + 1];
    __shared__ arc_shard_header_t glob;
    __shared__ int s_ok, s_last;
    const int tid = threadIdx.x;
    uint8_t *own = q.win[q.rank];
    asm volatile("griddepcontrol.wait;" ::: "memory");  // the local compare has completed

    // 1. publish (one thread of the grid)
    if (blockIdx.x == 0 && tid == 0) {
        unsigned long long *h = reinterpret_cast<unsigned long long *>(packet_at(own, q.cap, q.par));
        h[0] = q.n_local;
        h[1] = q.mirror->count;
        h[2] = q.mirror->max_abs_bits;
        h[3] = q.mirror->max_rel_bits;
        peer_fence_sys();  // header + the local report (previous kernels) before the flags
        for (int r = 0; r < q.p; ++r) st_release_sys(flag_slot(q.win[r], q.par, q.rank), q.s);
    }
    // 2. wait for every rank's flag in the own window
    if (tid == 0) {
        int ok = 1;
        const unsigned long long t0 = globaltimer();
        for (int r = 0; r < q.p && ok; ++r) {
            const unsigned long long *f = flag_slot(own, q.par, r);
            while (ld_acquire_sys(f) != q.s) {
                if (globaltimer() - t0 > kPeerTimeoutNs) {
                    ok = 0;
                    break;
                }
                __nanosleep(128);
            }
        }
        s_ok = ok;
    }
    __syncthreads();
    const bool ok = s_ok != 0;
    uint64_t total = 0;
    if (ok) {
        // 3. merge: headers from every window (P2P loads, not cached in L1)
        for (int r = tid; r < q.p; r += blockDim.x) {
            const unsigned long long *h = reinterpret_cast<const unsigned long long *>(packet_at(q.win[r], q.cap, q.par));
            hdr[r].n = ld_volatile(h);
            hdr[r].n_mismatch = ld_volatile(h + 1);
            hdr[r].max_abs_bits = ld_volatile(h + 2);
            hdr[r].max_rel_bits = ld_volatile(h + 3);
        }
        __syncthreads();
        if (tid == 0) {
            merge_plan_impl(hdr, q.p, q.max_report, plan, &glob);
            cum[0] = 0;
            for (int r = 0; r < q.p; ++r) cum[r + 1] = cum[r] + plan[r].contrib;
        }
        __syncthreads();
        total = q.dst ? cum[q.p] : 0;
        arc_mismatch_t *const dst = (q.dst_alias && total <= kDirectDyn) ? q.dst_alias : q.dst;
        for (uint64_t gi = (uint64_t)blockIdx.x * blockDim.x + tid; gi < total;
             gi += (uint64_t)gridDim.x * blockDim.x) {
            int lo = 0, hi = q.p;  // last r with cum[r] <= gi
            while (hi - lo > 1) {
                const int mid = (lo + hi) >> 1;
                if (cum[mid] <= gi) lo = mid; else hi = mid;
            }
            const uint64_t j = gi - cum[lo];
            const unsigned long long *src = reinterpret_cast<const unsigned long long *>(
                packet_at(q.win[lo], q.cap, q.par) + sizeof(arc_shard_header_t) + j * sizeof(arc_mismatch_t));
            arc_mismatch_t e;
            e.index = ld_volatile(src) + plan[lo].index_offset;
            e.out_bits = ld_volatile(src + 1);
            e.ref_bits = ld_volatile(src + 2);
            dst[plan[lo].prefix + j] = e;
        }
    }
    // 4. completion: the last block publishes the global header, then the word
    __syncthreads();
    if (tid == 0) {
        if (!ok) q.out[1].n = 1;  // status: timed out
        // gpu-scope release: the last block's system fence below is cumulative
        // (entries written to a pinned host report included)
        peer_fence_gpu();
        const unsigned long long prev = atomicAdd(q.done, 1ull);
        s_last = (prev - q.done_base) == (unsigned long long)(gridDim.x - 1);
    }
    __syncthreads();
    if (s_last && tid == 0) {
        peer_fence_gpu();
        if (ok) q.out[0] = glob;
        peer_fence_sys();
        *(volatile unsigned long long *)q.done_flag = q.seq;
    }
}

// ------------------------------------------------------------------- host
#define CK(call)                                                  \
    do {                                                          \
        cudaError_t e_ = (call);                                  \
        if (e_ != cudaSuccess) return cuda_fail(e_, #call);       \
    } while (0)

void peer_finalize(Ctx &c) {
    for (int r = 0; r < kMaxRanks; ++r)
        if (c.peer_map[r]) {
            cudaIpcCloseMemHandle(c.peer_map[r]);
            c.peer_map[r] = nullptr;
        }
    if (c.win) cudaFree(c.win);
    if (c.win_table) cudaFree(c.win_table);
    if (c.mirror) cudaFree(c.mirror);
    if (c.peer_out_host) cudaFreeHost(c.peer_out_host);
    c.win = nullptr;
    c.win_table = nullptr;
    c.mirror = nullptr;
    c.peer_out_host = c.peer_out_dev = nullptr;
    c.peer_ready = false;
}

// The sharded compare over the peer windows: local K1 into the own window,
// then one exchange+merge kernel, then one wait.
int peer_compare(Ctx &c, const arc_verify_region_t &r, arc_verify_result_t *result) {
    int st = validate_region(r.out, r.ref, r.n, r.dtype, r.abs_tol, r.rel_tol, r.max_report, result);
    if (st) return st;
    const unsigned long long s = ++c.coll_seq;
    const int par = (int)(s & 1);
    arc_mismatch_t *entries =
        reinterpret_cast<arc_mismatch_t *>(packet_at(c.win, c.win_cap, par) + sizeof(arc_shard_header_t));
    if (r.n == 0) CK(cudaMemsetAsync(c.mirror, 0, sizeof(Acc), c.stream));
    // local a1-a6 on the shard, enqueue only; the report goes to the own window
    arc_verify_result_t local;
    memset(&local, 0, sizeof(local));
    local.report = entries;
    c.defer_wait = true;
    c.mirror_next = c.mirror;
    st = run_local(c, &r, 1, &local, &entries, false, nullptr);
    c.defer_wait = false;
    c.mirror_next = nullptr;
    if (st) return st;
    // global report target
    arc_mismatch_t *dst = nullptr;
    bool host_report = false;
    if (r.max_report > 0) {
        st = report_target(c, result, r.max_report, &dst, &host_report);
        if (st) return st;
    }
    c.peer_out_host[1].n = 0;  // status
    PeerParams q;
    q.win = c.win_table;
    q.rank = c.rank;
    q.p = c.nranks;
    q.par = par;
    q.s = s;
    q.n_local = r.n;
    q.max_report = r.max_report;
    q.cap = c.win_cap;
    q.mirror = c.mirror;
    q.dst = dst;
    // a sparse global report goes straight into a pinned caller buffer
    q.dst_alias = host_report ? static_cast<arc_mismatch_t *>(pinned_device_alias(result->report)) : nullptr;
    q.out = c.peer_out_dev;
    q.done = c.counters + 5;
    q.done_base = c.peer_done_base;
    q.done_flag = c.flag_dev;
    q.seq = ++c.seq;
    // a few blocks: the merge moves <= max_report x 24 B, mostly a handful
    const uint64_t work = std::min<uint64_t>(r.max_report, 1ull << 40);
    const int grid = (int)std::max<uint64_t>(1, std::min<uint64_t>(32, (work + 2047) / 2048));
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(grid);
    cfg.blockDim = dim3(256);
    cfg.stream = c.stream;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    at[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = at;
    cfg.numAttrs = c.pdl ? 1 : 0;
    CK(cudaLaunchKernelEx(&cfg, arcv_peer_kernel, q));
    c.launches++;
    c.peer_done_base += (unsigned long long)grid;
    st = wait_results(c);
    if (st) return st;
    if (c.peer_out_host[1].n != 0) {
        set_error("peer exchange timed out (collective sequence %llu): a rank did not arrive", s);
        return ARC_E_CUDA;
    }
    fill_result(c.peer_out_host[0], r.max_report, result);
    if (host_report && result->n_reported && !(q.dst_alias && result->n_reported <= kDirectDyn)) {
        CK(cudaMemcpyAsync(result->report, dst, result->n_reported * sizeof(arc_mismatch_t), cudaMemcpyDeviceToHost,
                           c.stream));
        CK(cudaStreamSynchronize(c.stream));
    }
    return ARC_OK;
}

}  // namespace arcv

using namespace arcv;

extern "C" {

int arc_verify_peer_export(uint64_t max_report_cap, void *handle) {
    if (!g_ctx) return ARC_E_NOINIT;
    Ctx &c = *g_ctx;
    if (!handle || c.nranks > kMaxRanks || max_report_cap > (1ull << 36)) {
        set_error("peer_export: handle must be non-NULL, nranks <= %d, cap <= 2^36", kMaxRanks);
        return ARC_E_INVAL;
    }
    peer_finalize(c);
    const size_t bytes = kFlagBytes + 2 * packet_stride(max_report_cap);
    cudaError_t e = cudaMalloc(&c.win, bytes);
    if (e != cudaSuccess) {
        cudaGetLastError();
        set_error("cudaMalloc(peer window, %zu B)", bytes);
        return ARC_E_NOMEM;
    }
    CK(cudaMemset(c.win, 0, kFlagBytes));
    c.win_bytes = bytes;
    c.win_cap = max_report_cap;
    if (!c.mirror) {
        e = cudaMalloc(&c.mirror, sizeof(Acc));
        if (e != cudaSuccess) { cudaGetLastError(); set_error("cudaMalloc(mirror)"); return ARC_E_NOMEM; }
    }
    if (!c.peer_out_host) {
        e = cudaHostAlloc(reinterpret_cast<void **>(&c.peer_out_host), 2 * sizeof(arc_shard_header_t),
                          cudaHostAllocMapped);
        if (e != cudaSuccess) { cudaGetLastError(); set_error("cudaHostAlloc(peer out)"); return ARC_E_NOMEM; }
        CK(cudaHostGetDevicePointer(reinterpret_cast<void **>(&c.peer_out_dev), c.peer_out_host, 0));
    }
    cudaIpcMemHandle_t h;
    CK(cudaIpcGetMemHandle(&h, c.win));
    static_assert(sizeof(h) == 64, "cudaIpcMemHandle_t is 64 bytes");
    memcpy(handle, &h, sizeof(h));
    c.coll_seq = 0;
    return ARC_OK;
}

int arc_verify_peer_open(const void *handles) {
    if (!g_ctx) return ARC_E_NOINIT;
    Ctx &c = *g_ctx;
    if (!handles || !c.win) {
        set_error("peer_open: call arc_verify_peer_export first and pass nranks handles");
        return ARC_E_INVAL;
    }
    uint8_t *ptrs[kMaxRanks];
    for (int r = 0; r < c.nranks; ++r) {
        if (r == c.rank) {
            ptrs[r] = c.win;
            continue;
        }
        cudaIpcMemHandle_t h;
        memcpy(&h, static_cast<const uint8_t *>(handles) + 64 * (size_t)r, 64);
        void *p = nullptr;
        cudaError_t e = cudaIpcOpenMemHandle(&p, h, cudaIpcMemLazyEnablePeerAccess);
        if (e != cudaSuccess) {
            cudaGetLastError();
            set_error("cudaIpcOpenMemHandle(rank %d): %s", r, cudaGetErrorString(e));
            return ARC_E_UNSUPPORTED;
        }
        c.peer_map[r] = p;
        ptrs[r] = static_cast<uint8_t *>(p);
    }
    if (!c.win_table) {
        cudaError_t e = cudaMalloc(&c.win_table, kMaxRanks * sizeof(uint8_t *));
        if (e != cudaSuccess) { cudaGetLastError(); set_error("cudaMalloc(window table)"); return ARC_E_NOMEM; }
    }
    CK(cudaMemcpy(c.win_table, ptrs, c.nranks * sizeof(uint8_t *), cudaMemcpyHostToDevice));
    c.peer_ready = true;
    c.sharded = true;
    return ARC_OK;
}

}  // extern "C"
