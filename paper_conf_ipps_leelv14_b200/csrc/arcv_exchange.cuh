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

// Ring forwarding of large global reports: the entries of a
// contributing rank travel q -> q+1 -> ... -> q-1 in chunks of kRingChunk
// entries instead of every rank pulling them from q's window (which makes q's
// NVLink egress carry (p - 1) x the report).  Used when p >= 3 and the global
// report holds at least kRingMin entries; below that one hop from the owner is
// faster than a pipeline.  kRingGroups block groups keep that many chunks in
// flight per rank.
constexpr uint64_t kRingChunk = 1ull << 14;   // entries (384 KB)
constexpr uint64_t kRingMin = 1ull << 17;     // entries (3 MB)
constexpr int kRingGroups = 8;

__host__ __device__ inline uint64_t ring_chunks_max(uint64_t cap) { return cap / kRingChunk + kMaxRanks + 1; }
__host__ __device__ inline size_t ring_flag_bytes(uint64_t cap) {
    return ((size_t)ring_chunks_max(cap) * sizeof(unsigned long long) + 127) & ~(size_t)127;
}
__host__ __device__ inline size_t packet_stride(uint64_t cap) {
    return (sizeof(arc_shard_header_t) + (size_t)cap * sizeof(arc_mismatch_t) + 127) & ~(size_t)127;
}
// Window layout (identical on every rank; all ranks use the same cap):
//   [flags: 2 parities x kMaxRanks u64] [ring chunk flags: ring_chunks_max(cap) u64]
//   [packet parity 0] [packet parity 1] [forward area: cap entries]
__host__ __device__ inline unsigned long long *flag_slot(uint8_t *win, int par, int r) {
    return reinterpret_cast<unsigned long long *>(win) + (size_t)par * kMaxRanks + r;
}
__host__ __device__ inline unsigned long long *ring_flag(uint8_t *win, uint64_t c) {
    return reinterpret_cast<unsigned long long *>(win + kFlagBytes) + c;
}
__host__ __device__ inline uint8_t *packet_at(uint8_t *win, uint64_t cap, int par) {
    return win + kFlagBytes + ring_flag_bytes(cap) + (size_t)par * packet_stride(cap);
}
__host__ __device__ inline arc_mismatch_t *forward_area(uint8_t *win, uint64_t cap) {
    return reinterpret_cast<arc_mismatch_t *>(win + kFlagBytes + ring_flag_bytes(cap) + 2 * packet_stride(cap));
}
__host__ __device__ inline size_t window_bytes(uint64_t cap) {
    return kFlagBytes + ring_flag_bytes(cap) + 2 * packet_stride(cap) + (size_t)cap * sizeof(arc_mismatch_t);
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
__device__ __forceinline__ uint64_t warp_sum_u64_x(uint64_t v) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    return v;
}

// Block-private scratch of the exchange (~18.5 KB): static in the exchange
// kernel, carved from the (then free) stage memory in K1.
struct ExShared {
    arc_shard_header_t hdr[kMaxRanks];
    arc_shard_plan_t plan[kMaxRanks];
    uint64_t cum[kMaxRanks + 1];
    uint64_t cbase[kMaxRanks + 1];  // ring mode: first chunk id of each contributing rank
    arc_shard_header_t glob;
    unsigned long long deadline;
    int ok, last, go[2];
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

// Spin (thread 0) until *f == s or the call's deadline passes; false on timeout.
__device__ __forceinline__ bool wait_flag(const unsigned long long *f, unsigned long long s,
                                          unsigned long long deadline) {
    while (ld_acquire_sys(f) != s) {
        if (globaltimer() > deadline) return false;
        __nanosleep(64);
    }
    return true;
}

// Copy entries [j0, j1) of source rank `src`'s contribution (local positions
// within its contribution) from `from` -- the source's packet entries (local
// indices: `add` = the source's index offset) or a forwarding rank's area
// (global entries: add = 0) -- to `to` (and `fwd`, if not null), word by word
// (3 u64 per entry; coalesced 8-byte accesses).  Returns the bytes read.
__device__ __forceinline__ uint64_t copy_entries(const unsigned long long *from, uint64_t add,
                                                 unsigned long long *to, unsigned long long *fwd, uint64_t w0,
                                                 uint64_t w1, int tid) {
    for (uint64_t w = w0 + tid; w < w1; w += 256) {
        unsigned long long v = ld_volatile(from + w);
        if (w % 3 == 0) v += add;
        to[w] = v;
        if (fwd) fwd[w] = v;
    }
    return tid == 0 ? (w1 - w0) * 8 : 0;  // counted once per block
}

// Steps 2-4 of the exchange for this block (`tid` in 0..255, every thread of
// the 256 calls it).  `done_base`: the host-tracked base of q.done.
__device__ __forceinline__ void peer_exchange_body(const PeerParams &q, int tid, ExShared &sh) {
    uint8_t *own = q.win[q.rank];
    // 2. wait for every rank's flag in the own window (bounded)
    if (tid == 0) {
        int ok = 1;
        sh.deadline = globaltimer() + kPeerTimeoutNs;
        for (int r = 0; r < q.p && ok; ++r)
            if (!wait_flag(flag_slot(own, q.par, r), q.s, sh.deadline)) ok = 0;
        sh.ok = ok;
    }
    exchange_bar();
    // ring chunk counters of the other parity (the previous call's, complete on
    // this rank): cleared by every call, whatever its mode, for the next one
    {
        uint32_t *cnt_old = q.ring_cnt + (size_t)(q.par ^ 1) * q.ring_cnt_n;
        for (uint64_t i = (uint64_t)blockIdx.x * 256 + tid; i < q.ring_cnt_n; i += (uint64_t)gridDim.x * 256)
            cnt_old[i] = 0u;
    }
    if (sh.ok) {
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
            sh.cbase[0] = 0;
            for (int r = 0; r < q.p; ++r) {
                sh.cum[r + 1] = sh.cum[r] + sh.plan[r].contrib;
                sh.cbase[r + 1] = sh.cbase[r] + (sh.plan[r].contrib + kRingChunk - 1) / kRingChunk;
            }
        }
        exchange_bar();
        const uint64_t total = q.dst ? sh.cum[q.p] : 0;
        uint64_t remote_bytes[2] = {0, 0};  // [0]: pulled from owners' packets, [1]: from forwarding ranks
        if (q.p >= 3 && total >= kRingMin) {
            // ---- ring forwarding (every rank computes the same plan and chunk list)
            const uint64_t nc = sh.cbase[q.p];
            uint32_t *cnt = q.ring_cnt + (size_t)q.par * q.ring_cnt_n;
            uint32_t it = 0;
            const int W = (int)gridDim.x < kRingGroups ? (int)gridDim.x : kRingGroups;
            const int grp = (int)blockIdx.x % W;
            const uint32_t gsz = (gridDim.x - (uint32_t)grp + W - 1) / W;  // blocks in my group
            const uint32_t gi = blockIdx.x / W;                            // my index in it
            unsigned long long *dstw = reinterpret_cast<unsigned long long *>(q.dst);
            const int succ = (q.rank + 1) % q.p, pred = (q.rank + q.p - 1) % q.p;
            for (uint64_t c = grp; c < nc; c += W, ++it) {
                int src = 0;  // contributing rank of chunk c: last r with cbase[r] <= c
                {
                    int lo = 0, hi = q.p;
                    while (hi - lo > 1) {
                        const int mid = (lo + hi) >> 1;
                        if (sh.cbase[mid] <= c) lo = mid; else hi = mid;
                    }
                    src = lo;
                }
                const int k = (q.rank - src + q.p) % q.p;  // my distance from the source on the ring
                const uint64_t j0 = (c - sh.cbase[src]) * kRingChunk;
                const uint64_t jn = sh.plan[src].contrib - j0 < kRingChunk ? sh.plan[src].contrib - j0 : kRingChunk;
                // my block's slice of the chunk
                const uint64_t per = (jn + gsz - 1) / gsz;
                const uint64_t a = j0 + (uint64_t)gi * per < j0 + jn ? j0 + (uint64_t)gi * per : j0 + jn;
                const uint64_t b = a + per < j0 + jn ? a + per : j0 + jn;
                const uint64_t pre = sh.plan[src].prefix;
                const unsigned long long *pk = reinterpret_cast<const unsigned long long *>(
                    packet_at(q.win[src], q.cap, q.par) + sizeof(arc_shard_header_t));
                if (k == 0) {  // the source: its own entries, locally
                    copy_entries(pk, sh.plan[src].index_offset, dstw + 3 * pre, nullptr, 3 * a, 3 * b, tid);
                    continue;
                }
                if (k >= 2) {  // the predecessor forwards the chunk: wait for its flag
                    // (result in a slot by iteration parity: thread 0 may write the
                    // next iteration's slot before a slow thread read this one)
                    if (tid == 0) {
                        const bool got = wait_flag(ring_flag(own, c), q.s, sh.deadline);
                        if (!got) sh.ok = 0;
                        sh.go[it & 1] = got;
                    }
                    exchange_bar();
                    if (!sh.go[it & 1]) break;
                }
                const bool forward = k < q.p - 1;
                unsigned long long *fw = forward ? reinterpret_cast<unsigned long long *>(
                                                       forward_area(own, q.cap) + pre) : nullptr;
                if (k == 1) {
                    remote_bytes[0] += copy_entries(pk, sh.plan[src].index_offset, dstw + 3 * pre, fw, 3 * a,
                                                    3 * b, tid);
                } else {
                    const unsigned long long *pf = reinterpret_cast<const unsigned long long *>(
                        forward_area(q.win[pred], q.cap) + pre);
                    remote_bytes[1] += copy_entries(pf, 0, dstw + 3 * pre, fw, 3 * a, 3 * b, tid);
                }
                if (forward) {
                    // the group's last block to finish the chunk tells the successor
                    exchange_bar();
                    if (tid == 0) {
                        peer_fence_gpu();
                        if (atomicAdd(cnt + c, 1u) == gsz - 1) {
                            peer_fence_sys();
                            st_release_sys(ring_flag(q.win[succ], c), q.s);
                        }
                    }
                }
            }
        } else {
            // ---- pull from the owners' windows (sparse reports, p <= 2)
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
                if (lo != q.rank) remote_bytes[0] += sizeof(arc_mismatch_t);
            }
        }
        // bytes this rank read from peer windows (arc_verify_peer_stats)
        if (q.stats) {
            const uint64_t b0 = warp_sum_u64_x(remote_bytes[0]), b1 = warp_sum_u64_x(remote_bytes[1]);
            if ((tid & 31) == 0 && (b0 | b1)) {
                atomicAdd(q.stats, (unsigned long long)b0);
                atomicAdd(q.stats + 1, (unsigned long long)b1);
            }
        }
    }
    // 4. completion: the last block publishes the global header, then the word
    exchange_bar();
    if (tid == 0) {
        if (!sh.ok) q.out[1].n = 1;  // status: timed out
        // gpu-scope release: the last block's system fence below is cumulative
        // (entries written to a pinned host report included)
        peer_fence_gpu();
        const unsigned long long prev = atomicAdd(q.done, 1ull);
        sh.last = (prev - q.done_base) == (unsigned long long)(gridDim.x - 1);
    }
    exchange_bar();
    if (sh.last && tid == 0) {
        peer_fence_gpu();
        if (sh.ok) q.out[0] = sh.glob;
        peer_fence_sys();
        *(volatile unsigned long long *)q.done_flag = q.seq;
    }
}

}  // namespace arcv
