// arcv_types.h -- workspace / launch descriptors shared by host and device code.
#pragma once
#include <cstdint>

#include "arc_verify.h"

namespace arcv {

constexpr int kTileBytes = 16384;                   // per array per tile
constexpr int kSlack = 32;                          // misaligned-window slack
constexpr int kStageArrayBytes = kTileBytes + kSlack;
constexpr int kStageBytes = 2 * kStageArrayBytes;   // out + ref
constexpr int kConsumerWarps = 8;
constexpr int kConsumerThreads = kConsumerWarps * 32;
constexpr int kThreads = kConsumerThreads + 32;     // + producer warp
constexpr int kVecPerThread = kTileBytes / 16 / kConsumerThreads;  // 4
constexpr int kMaxInlineSegs = 16;                 // regions passed as kernel parameters (C3: 12)
constexpr int kAllDtypes = 31;                      // K1 dtype-set masks: bit 1 << ARC_*
constexpr int kDtmFloatI32 = (1 << ARC_F32) | (1 << ARC_F64) | (1 << ARC_I32);  // batches without i64 / u8
constexpr int kGroupTiles = 256;                    // tiles per group counter
constexpr int kPoolCap = 2048;                      // report phase, pool path: max listed nonzero tiles
#ifndef ARCV_DIRECT_DYN
#define ARCV_DIRECT_DYN 4096
#endif
constexpr uint64_t kDirectDyn = ARCV_DIRECT_DYN;               // sparse reports: written directly into pinned host memory
constexpr uint64_t kDirectBit = 1ull << 63;         // report-phase tile prefix flag: entries go to report_alias
// Pool path (<= kPoolCap reported tiles): a denser pinned-host report is still
// written by the kernel itself, each dense tile staged in shared memory and
// stored as coalesced 8-byte words, up to kDirectDense entries; beyond that
// HBM staging + one D2H.
constexpr uint64_t kDirectDense = 1ull << 18;
constexpr uint64_t kStagedMin = 64;                 // tiles with more entries: staged, coalesced writes
constexpr uint64_t kPinStage = 1ull << 16;          // pageable report: library pinned staging per region
constexpr uint64_t kRoutePool = 1ull;               // Acc.pad of a published slot: the report took the pool path
static_assert(kVecPerThread == 4, "packed-scan layout assumes 4 vectors per thread");
static_assert(kGroupTiles == kConsumerThreads, "the report phase scans one group per block pass");

// Tile scheduling of multi-segment launches (batches): guided self-scheduling
// (a producer takes a run of consecutive tiles, ~remaining / (kGuide x grid),
// 1..kChunkMax) instead of one ticket per tile, so a CTA meets each region in
// longer runs and pays the per-region, per-CTA costs (accumulator flush, filter
// seeding and warm-up) fewer times: 12 fp32 regions 121 -> 112 us, C3 138 ->
// 134 us.  Single-segment launches keep one tile per ticket (runs measured
// 1-2 % slower there).  -DARCV_GUIDED=0: never guided (A/B builds).
#ifndef ARCV_GUIDED
#define ARCV_GUIDED 1
#endif
#ifndef ARCV_CHUNK_MAX
#define ARCV_CHUNK_MAX 16  // round 2: 8 -> 16, C3 batch 133.3 -> 129.7 us (profiles/r02g_ab_chunk.log)
#endif
constexpr uint64_t kChunkMax = ARCV_CHUNK_MAX, kGuide = 4;

constexpr uint32_t kFlagProbe = 2u;       // Params.flags: stream only, no predicate (read probe)
constexpr uint32_t kEnvFlagMask = 1u | 8u;  // ARCV_FLAGS bits honoured: 1 proxy fence, 8 stream-sync waits
constexpr uint32_t kSegBaseFromAcc = 1u;  // chunk of a streamed region: prefix base = acc count - own total
constexpr uint32_t kSegReportHost = 2u;   // `report` is (mapped) host memory (ARCV_WRITER_SYS diagnostic)

// One contiguous piece of one region (a whole region, or one chunk of a region
// streamed from host memory).
struct Seg {
    const uint8_t *out;
    const uint8_t *ref;
    uint64_t n;             // elements in this segment
    uint64_t tile_begin;    // launch-local index of the segment's first tile
    uint64_t slot_begin;    // per-tile count slot of the first tile
    uint64_t group_begin;   // group counter of the first tile's group
    uint64_t index_base;    // global element index of element 0
    double abs_tol, rel_tol;
    uint64_t max_report;    // report capacity / truncation for the region (0 = count only)
    arc_mismatch_t *report; // device pointer, entries [0, max_report)
    arc_mismatch_t *report_alias;  // device alias of the caller's pinned host report, or nullptr:
                                   // used instead of `report` when direct_route() holds (then
                                   // the host skips the D2H copy)
    uint64_t alias_cap;            // entries available at report_alias
    uint32_t acc_slot;
    uint32_t dtype;
    uint32_t flags;
    float at_rd, rt_rd;     // fp32 lower bounds of abs_tol / rel_tol (fp32 pre-filter)
    uint32_t cflags;        // ARC_CHECK_* (N2)
    double minv, lo, hi;    // check parameters
};

struct Acc {  // per-region accumulators / result slot, 32 bytes
    unsigned long long count;
    unsigned long long max_abs_bits;
    unsigned long long max_rel_bits;
    unsigned long long pad;  // published slot: slot_tag(seq, route, ...) (route: kRoutePool or 0)
};

// A published result slot validates itself: pad = ((seq << 1) | route) xor a
// 64-bit hash of the three result words.  The host accepts a slot only when
// the tag decodes to the call's sequence number, so a slot written over PCIe
// without a system fence (clean and count-only calls, which wrote no report
// entries to host memory) is never read torn or stale: the host re-reads
// until the whole slot has landed (a torn read passes with probability 2^-63).
__host__ __device__ inline uint64_t slot_mix(uint64_t z) {
    z ^= z >> 30;
    z *= 0xBF58476D1CE4E5B9ull;
    z ^= z >> 27;
    z *= 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}
__host__ __device__ inline uint64_t slot_tag(uint64_t seq, uint64_t route, uint64_t count, uint64_t abs_bits,
                                             uint64_t rel_bits) {
    return ((seq << 1) | route) ^ slot_mix(count ^ slot_mix(abs_bits ^ slot_mix(rel_bits ^ 0x5BD1E9955BD1E995ull)));
}

// Whether a region's report entries are written by the kernel straight into
// the pinned host buffer behind report_alias (no D2H copy).  One definition,
// applied by the report phase and -- with `pool` read back from the published
// slot -- by the host to decide whether it still has to copy.
__host__ __device__ inline bool direct_route(bool has_alias, uint32_t seg_flags, uint64_t count, uint64_t max_report,
                                             uint64_t alias_cap, bool pool) {
    const uint64_t entries = count < max_report ? count : max_report;
    return has_alias && !(seg_flags & kSegBaseFromAcc) && entries <= alias_cap &&
           (count <= kDirectDyn || (pool && count <= kDirectDense));
}

// The sharded exchange over peer windows (arcv_exchange.cuh): one call's
// parameters, used by the exchange kernel and by K1's fused exchange.
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
    uint32_t *ring_cnt;             // [2 parities][ring_cnt_n] per-chunk block counters (ring mode; local HBM)
    uint64_t ring_cnt_n;
    unsigned long long *stats;      // [2] monotonic: bytes read from owners' packets / forwarding ranks
};

struct Params {
    const Seg *segs;          // device table, or nullptr -> ParamsN::inline_segs
    uint32_t n_segs;
    uint32_t n_acc;
    uint64_t total_tiles;
    unsigned long long *ticket;
    unsigned long long ticket_base;
    unsigned long long *done;
    unsigned long long done_base;
    uint32_t *tile_cnt;       // per-tile mismatch counts (zero between calls)
    uint32_t *group_cnt;      // per-group counts of this launch
    uint32_t *group_zero;     // the other parity buffer, zeroed by K1 for the next launch
    uint64_t n_group_zero;
    uint64_t *active;         // report-phase active-tile list: {seg << 40 | tile, prefix}
    uint32_t *active_cnt;     // this launch's list length
    uint32_t *active_cnt_zero;  // the other parity, zeroed by K1 for the next launch
    uint64_t *nz_list;        // K1 -> report phase pool: {seg << 40 | tile, count} of nonzero tiles
    uint32_t *nz_cnt;         // this launch's pool length (may exceed kPoolCap: overflow)
    uint32_t *nz_cnt_zero;    // the other parity
    int k2;                   // some segment wants a report (report phase: fused, or K2 follows)
    int fused;                // K1 runs the report phase itself (cooperative launch; no K2)
    unsigned long long *gbar; // report-phase grid barrier counter (monotonic)
    unsigned long long gbar_base;
    Acc *acc;
    Acc *result;
    unsigned long long *done_flag;  // mapped host word: seq is stored when the call's results are final
    unsigned long long seq;
    Acc *mirror;                    // optional device copy of the published result slots (peer exchange)
    uint32_t report_host;           // some report lives in pinned host memory (system-scope fences)
    int finalize;
    uint32_t flags;
    int guided;                     // guided self-scheduling of tiles (multi-segment launches)
    int xfused;                     // sharded call: K1's CTAs run the exchange after the local result
    PeerParams x;                   // its parameters (xfused only)
};

// The kernels' parameter block: Params plus NSEG inline segments.  The launch
// cost grows with the parameter bytes (measured: C1 per call 30.0 -> 27.1 us
// with 1 instead of 16 inline segments), so single-region calls -- the common
// case -- use NSEG = 1 and batches of up to kMaxInlineSegs regions NSEG = 16;
// larger batches pass a device table (segs) with NSEG = 1.
template <int NSEG>
struct ParamsN : Params {
    Seg inline_segs[NSEG];
};

static_assert(sizeof(ParamsN<kMaxInlineSegs>) <= 4096, "kernel parameters stay within the classic 4 KB limit");

struct StageInfo {
    uint64_t tile;        // launch-local tile, ~0 = no more work
    uint64_t elem_begin;  // segment-local index of the tile's first element
    uint32_t seg;
    uint32_t count;       // valid elements in the tile
    uint32_t off_o, off_r;
};

__host__ __device__ constexpr uint32_t elem_size(uint32_t dt) {
    return dt == ARC_F64 || dt == ARC_I64 ? 8u : (dt == ARC_U8 ? 1u : 4u);
}
__host__ __device__ constexpr uint64_t tile_elems(uint32_t dt) { return kTileBytes / elem_size(dt); }

}  // namespace arcv
