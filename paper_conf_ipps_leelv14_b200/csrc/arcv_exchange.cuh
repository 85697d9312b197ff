// arcv_exchange.cuh -- the device side of the sharded exchange over peer
// memory, shared by the
// stand-alone exchange kernel (arcv_peer.cu) and the fused exchange that runs in
// K1's tail (arcv_device.cuh).  The protocol, the window layout and the reuse
// rules are described at the top of arcv_peer.cu.
//
//   peer_publish_header : the rank's leader writes its 32-byte header into its
//                         own window and releases flag [par][rank] in EVERY
//                         window (st.release.sys over NVLink / NVSwitch).
//   peer_exchange_body  : every block waits for the p flags of its own window,
//                         rebuilds the merge plan (arcv_merge.h, the one
//                         definition), copies its share of the contributing
//                         entries from the peers' windows into the global
//                         report, and the last block writes the global header
//                         to mapped host memory and then the completion word.
// Participating threads per block: 256, synchronised on named barrier 1 (the
// consumer warps of K1; all threads of the exchange kernel).
#pragma once
#include <cstdint>

#include "arc_verify.h"
#include "arcv_merge.h"
#include "arcv_types.h"

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

__device__ __forceinline__ void st_release_sys(unsigned long long *p, unsigned long long v) {
    asm volatile("st.release.sys.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ unsigned long long ld_acquire_sys(const unsigned long long *p) {
    unsigned long long v;
    asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
// message-passing fences (no fence.sc needed)
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
__device__ __forceinline__ void exchange_bar() { asm volatile("bar.sync 1, 256;" ::: "memory"); }

// Block-private scratch of the exchange (~16.5 KB): static in the exchange
// kernel, carved from the (then free) stage memory in K1.
struct ExShared {
    arc_shard_header_t hdr[kMaxRanks];
    arc_shard_plan_t plan[kMaxRanks];
    uint64_t cum[kMaxRanks + 1];
    arc_shard_header_t glob;
    int ok, last;
};

// The rank's header {n_local, count, max_abs_bits, max_rel_bits} into its own
// window, then the call's sequence number into flag [par][rank] of every
// window.  One thread per rank and call.  The system-scope fence orders the
// header and the local report (written earlier by this grid or a previous
// kernel) before the flags.
__device__ __forceinline__ void peer_publish_header(const PeerParams &q, unsigned long long count,
                                                    unsigned long long abs_bits, unsigned long long rel_bits) {
    uint8_t *own = q.win[q.rank];
    unsigned long long *h = reinterpret_cast<unsigned long long *>(packet_at(own, q.cap, q.par));
    h[0] = q.n_local;
    h[1] = count;
    h[2] = abs_bits;
    h[3] = rel_bits;
    peer_fence_sys();
    for (int r = 0; r < q.p; ++r) st_release_sys(flag_slot(q.win[r], q.par, q.rank), q.s);
}

// Steps 2-4 of the exchange for this block (`tid` in 0..255, every thread of
// the 256 calls it).  `done_base`: the host-tracked base of q.done.
__device__ __forceinline__ void peer_exchange_body(const PeerParams &q, int tid, ExShared &sh) {
    uint8_t *own = q.win[q.rank];
    // 2. wait for every rank's flag in the own window (bounded)
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
                __nanosleep(64);
            }
        }
        sh.ok = ok;
    }
    exchange_bar();
    const bool ok = sh.ok != 0;
    if (ok) {
        // 3. merge: headers from every window (P2P loads, not cached in L1)
        for (int r = tid; r < q.p; r += 256) {
            const unsigned long long *h = reinterpret_cast<const unsigned long long *>(packet_at(q.win[r], q.cap, q.par));
            sh.hdr[r].n = ld_volatile(h);
            sh.hdr[r].n_mismatch = ld_volatile(h + 1);
            sh.hdr[r].max_abs_bits = ld_volatile(h + 2);
            sh.hdr[r].max_rel_bits = ld_volatile(h + 3);
        }
        exchange_bar();
        if (tid == 0) {
            merge_plan_impl(sh.hdr, q.p, q.max_report, sh.plan, &sh.glob);
            sh.cum[0] = 0;
            for (int r = 0; r < q.p; ++r) sh.cum[r + 1] = sh.cum[r] + sh.plan[r].contrib;
        }
        exchange_bar();
        const uint64_t total = q.dst ? sh.cum[q.p] : 0;
        // a sparse global report goes straight into the caller's pinned buffer
        arc_mismatch_t *const dst = (q.dst_alias && total <= kDirectDyn) ? q.dst_alias : q.dst;
        for (uint64_t gi = (uint64_t)blockIdx.x * 256 + tid; gi < total; gi += (uint64_t)gridDim.x * 256) {
            int lo = 0, hi = q.p;  // last r with cum[r] <= gi
            while (hi - lo > 1) {
                const int mid = (lo + hi) >> 1;
                if (sh.cum[mid] <= gi) lo = mid; else hi = mid;
            }
            const uint64_t j = gi - sh.cum[lo];
            const unsigned long long *src = reinterpret_cast<const unsigned long long *>(
                packet_at(q.win[lo], q.cap, q.par) + sizeof(arc_shard_header_t) + j * sizeof(arc_mismatch_t));
            arc_mismatch_t e;
            e.index = ld_volatile(src) + sh.plan[lo].index_offset;
            e.out_bits = ld_volatile(src + 1);
            e.ref_bits = ld_volatile(src + 2);
            dst[sh.plan[lo].prefix + j] = e;
        }
    }
    // 4. completion: the last block publishes the global header, then the word
    exchange_bar();
    if (tid == 0) {
        if (!ok) q.out[1].n = 1;  // status: timed out
        // gpu-scope release: the last block's system fence below is cumulative
        // (entries written to a pinned host report included)
        peer_fence_gpu();
        const unsigned long long prev = atomicAdd(q.done, 1ull);
        sh.last = (prev - q.done_base) == (unsigned long long)(gridDim.x - 1);
    }
    exchange_bar();
    if (sh.last && tid == 0) {
        peer_fence_gpu();
        if (ok) q.out[0] = sh.glob;
        peer_fence_sys();
        *(volatile unsigned long long *)q.done_flag = q.seq;
    }
}

}  // namespace arcv
