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
#include "arcv_exchange.cuh"
#include "arcv_internal.h"

namespace arcv {

// The stand-alone exchange kernel: a programmatic dependent of the local
// compare (K1), used when K1 did not run the exchange itself (empty or
// host-streamed shard, ARCV_FUSED_EXCHANGE=0).  Block 0 publishes the header
// from the local summary mirror; every block then runs the common body.
__global__ void __launch_bounds__(256) arcv_peer_kernel(const __grid_constant__ PeerParams q) {
    __shared__ ExShared sh;
    asm volatile("griddepcontrol.wait;" ::: "memory");  // the local compare has completed
    if (blockIdx.x == 0 && threadIdx.x == 0)
        peer_publish_header(q, q.mirror->count, q.mirror->max_abs_bits, q.mirror->max_rel_bits);
    peer_exchange_body(q, (int)threadIdx.x, sh);
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
    if (c.ring_cnt) cudaFree(c.ring_cnt);
    if (c.peer_stats) cudaFree(c.peer_stats);
    c.ring_cnt = nullptr;
    c.ring_cnt_n = 0;
    c.peer_stats = nullptr;
    c.win = nullptr;
    c.win_table = nullptr;
    c.mirror = nullptr;
    c.peer_out_host = c.peer_out_dev = nullptr;
    c.peer_ready = false;
}

// The sharded compare over the peer windows: local K1 into the own window and
// -- fused, the default -- the exchange in the same kernel's tail (K1 is then a
// cooperative launch: its CTAs wait for the peers' flags), else one
// exchange+merge kernel after it; then one wait.
int peer_compare(Ctx &c, const arc_verify_region_t &r, arc_verify_result_t *result) {
    int st = validate_region(r.out, r.ref, r.n, r.dtype, r.abs_tol, r.rel_tol, r.max_report, result);
    if (st) return st;
    const unsigned long long s = ++c.coll_seq;
    const int par = (int)(s & 1);
    arc_mismatch_t *entries =
        reinterpret_cast<arc_mismatch_t *>(packet_at(c.win, c.win_cap, par) + sizeof(arc_shard_header_t));
    if (r.n == 0) CK(cudaMemsetAsync(c.mirror, 0, sizeof(Acc), c.stream));
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
    q.done = c.counters + Ctx::kCtrPeerDone;
    q.done_base = c.peer_done_base;
    q.done_flag = c.flag_dev;
    q.seq = ++c.seq;
    q.ring_cnt = c.ring_cnt;
    q.ring_cnt_n = c.ring_cnt_n;
    q.stats = c.peer_stats;
    // the fused exchange needs a local launch: a non-empty, device-resident shard
    const bool want_fused = c.fused_exchange && r.n > 0 && classify(r.out, c.device) == PK_DEVICE &&
                            classify(r.ref, c.device) == PK_DEVICE;
    // local a1-a6 on the shard, enqueue only; the report goes to the own window
    arc_verify_result_t local;
    memset(&local, 0, sizeof(local));
    local.report = entries;
    c.defer_wait = true;
    c.mirror_next = c.mirror;
    c.x_next = want_fused ? &q : nullptr;
    c.x_taken = false;
    st = run_local(c, &r, 1, &local, &entries, false, nullptr);
    c.defer_wait = false;
    c.mirror_next = nullptr;
    c.x_next = nullptr;
    if (st) return st;
    if (!c.x_taken) {
        // blocks by the report size: a handful for the usual sparse report, one
        // per SM for a dense one (ring forwarding keeps kRingGroups chunks in flight)
        q.done_base = c.peer_done_base;
        const uint64_t work = std::min<uint64_t>(r.max_report, 1ull << 40);
        const int grid = (int)std::max<uint64_t>(1, std::min<uint64_t>((uint64_t)c.num_sms, (work + 2047) / 2048));
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
    }
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
    const size_t bytes = window_bytes(max_report_cap);
    cudaError_t e = cudaMalloc(&c.win, bytes);
    if (e != cudaSuccess) {
        cudaGetLastError();
        set_error("cudaMalloc(peer window, %zu B)", bytes);
        return ARC_E_NOMEM;
    }
    CK(cudaMemset(c.win, 0, kFlagBytes + ring_flag_bytes(max_report_cap)));  // call flags + ring chunk flags
    c.ring_cnt_n = ring_chunks_max(max_report_cap);
    e = cudaMalloc(&c.ring_cnt, 2 * c.ring_cnt_n * sizeof(uint32_t));
    if (e != cudaSuccess) { cudaGetLastError(); set_error("cudaMalloc(ring counters)"); return ARC_E_NOMEM; }
    CK(cudaMemset(c.ring_cnt, 0, 2 * c.ring_cnt_n * sizeof(uint32_t)));
    e = cudaMalloc(&c.peer_stats, 2 * sizeof(unsigned long long));
    if (e != cudaSuccess) { cudaGetLastError(); set_error("cudaMalloc(peer stats)"); return ARC_E_NOMEM; }
    CK(cudaMemset(c.peer_stats, 0, 2 * sizeof(unsigned long long)));
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

int arc_verify_peer_stats(uint64_t *bytes, int reset) {
    if (!g_ctx) return ARC_E_NOINIT;
    Ctx &c = *g_ctx;
    if (!bytes) { set_error("peer_stats: bytes is NULL"); return ARC_E_INVAL; }
    if (!c.peer_stats) {
        bytes[0] = bytes[1] = 0;
        return ARC_OK;
    }
    unsigned long long h[2];
    CK(cudaStreamSynchronize(c.stream));
    CK(cudaMemcpy(h, c.peer_stats, sizeof(h), cudaMemcpyDeviceToHost));
    bytes[0] = h[0];
    bytes[1] = h[1];
    if (reset) CK(cudaMemset(c.peer_stats, 0, sizeof(h)));
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
