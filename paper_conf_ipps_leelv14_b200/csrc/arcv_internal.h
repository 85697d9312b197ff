// arcv_internal.h -- library-private context and cross-file declarations.
#pragma once
#include <cuda_runtime.h>

#include <cstdint>

#include "arc_verify.h"
#include "arcv_merge.h"
#include "arcv_types.h"

namespace arcv {

enum PtrKind { PK_DEVICE, PK_HOST, PK_BAD };

struct Ctx {
    static constexpr int kNBuf = 2;                       // host-input chunk ring
    static constexpr size_t kChunkBytes = 64ull << 20;    // per array per chunk
    static constexpr int kMaxEv = 64;

    int device = 0;
    int rank = 0, nranks = 1;
    bool sharded = false;  // collective path (NCCL communicator), nranks >= 1
    int num_sms = 0, ctas_per_sm = 1, stages = 3, flags = 0;
    int k2_grid = 0;  // K2 (cooperative) grid: SMs x co-resident CTAs (<= 2)
    uint64_t direct_max = 0;  // pinned host reports up to this capacity: written by the kernel
    bool fused = true;  // report phase in K1's tail (cooperative K1), no K2 launch
    bool pdl = true;  // launch K2 / the exchange kernel as programmatic dependents (ARCV_PDL=0: off)
    bool dt_spec = true;  // single-region calls: K1 specialised for the region's dtype (ARCV_DT_SPEC=0: generic)
    bool sort_segs = true;  // batches: smallest regions' tiles first (ARCV_SORT_SEGS=0: listed order)
    cudaStream_t stream = nullptr;
    bool own_stream = false;
    cudaStream_t copy_stream = nullptr;

    // Device counter words (one 64-byte allocation; the map below is the only
    // place that assigns them -- every user goes through these indices):
    //   [kCtrTicket]    K1 tile tickets              (monotonic, host-tracked base)
    //   [kCtrDone]      finished K1/K2 CTAs          (monotonic, host-tracked base)
    //   [kCtrGbar]      report-phase grid barrier    (monotonic, host-tracked base)
    //   [kCtrActive]    2 x u32 active-list lengths  (by call parity)
    //   [kCtrPool]      2 x u32 pool lengths         (by call parity)
    //   [kCtrPeerDone]  peer-exchange finished blocks (monotonic, peer_done_base)
    //   [kCtrChecksum]  2 words: checksum sum / xor accumulators (zeroed per call)
    static constexpr int kCtrTicket = 0, kCtrDone = 1, kCtrGbar = 2, kCtrActive = 3, kCtrPool = 4,
                         kCtrPeerDone = 5, kCtrChecksum = 6, kCtrWords = 8;
    unsigned long long *counters = nullptr;
    unsigned long long ticket_base = 0, done_base = 0;

    uint32_t *tile_cnt = nullptr;      size_t tile_cnt_cap = 0;   // per-tile counts (kept zero)
    uint64_t *active = nullptr;        size_t active_cap = 0;     // report-phase active list (2 words / entry)
    uint32_t *active_cnt = nullptr;                               // [2] by parity
    uint64_t *nz_list = nullptr;                                  // K1 -> report-phase pool (kPoolCap entries)
    uint32_t *nz_cnt = nullptr;                                   // [2] by parity
    unsigned long long gbar_base = 0;
    uint32_t *group_cnt = nullptr;     size_t group_cap = 0;      // [2][group_cap], parity per K1
    int parity = 0;
    Acc *acc = nullptr;                size_t acc_cap = 0;
    unsigned long long *flag_host = nullptr, *flag_dev = nullptr;  // mapped completion word
    unsigned long long seq = 0;                                      // last finalize launch's number
    Acc *result_host = nullptr;        size_t result_host_cap = 0;   // mapped pinned
    Acc *result_dev = nullptr;                                       // its device alias
    Seg *seg_dev = nullptr;            size_t seg_dev_cap = 0;
    Seg *seg_host = nullptr;           size_t seg_host_cap = 0;
    cudaEvent_t ev_seg = nullptr;      // after the last segment-table copy
    bool seg_copy_pending = false;
    arc_mismatch_t *report_stage = nullptr; size_t report_stage_cap = 0;
    arc_mismatch_t *report_pin = nullptr;      // mapped pinned staging (sparse pageable reports)
    arc_mismatch_t *report_pin_dev = nullptr;  // its device alias
    size_t report_pin_cap = 0;

    void *chunk_buf[kNBuf][2] = {{nullptr, nullptr}, {nullptr, nullptr}};
    cudaEvent_t ev_copy[kNBuf] = {}, ev_free[kNBuf] = {};
    uint64_t h2d_bytes = 0;

    // timing (bench)
    bool timing = false;
    cudaEvent_t ev[kMaxEv][2] = {};
    int n_ev = 0;
    uint64_t launches = 0, timed_launches = 0;
    double timed_ms = 0.0;

    // sharded mode
    void *nccl_comm = nullptr;
    uint8_t *packet = nullptr;         size_t packet_cap = 0;     // bytes
    uint8_t *gathered = nullptr;       size_t gathered_cap = 0;   // bytes
    arc_shard_header_t *hdr_host = nullptr; size_t hdr_host_cap = 0;
    arc_shard_header_t *merge_dev = nullptr;                        // [1 + nranks] global + per-rank

    // peer-memory exchange (arcv_peer.cu): symmetric windows over NVLink P2P
    bool defer_wait = false;           // run_local: enqueue only (the exchange kernel follows)
    const PeerParams *x_next = nullptr;  // launch_segments: run this exchange in K1's tail (fused)
    bool x_taken = false;              // ... and it did (else the exchange kernel runs)
    bool fused_exchange = true;        // ARCV_FUSED_EXCHANGE=0: always the separate exchange kernel
    Acc *mirror_next = nullptr;        // launch_segments: device copy of the finalised slots
    Acc *mirror = nullptr;             // [1] device
    uint8_t *win = nullptr;            // own window (cudaMalloc, IPC-exported)
    size_t win_bytes = 0;
    uint64_t win_cap = 0;              // report entries per packet
    void *peer_map[kMaxRanks] = {};    // IPC-mapped peer windows (to close)
    uint8_t **win_table = nullptr;     // device [nranks] window pointers (own included)
    bool peer_ready = false;
    unsigned long long coll_seq = 0;   // collective calls made (flag value of the last)
    unsigned long long peer_done_base = 0;
    arc_shard_header_t *peer_out_host = nullptr, *peer_out_dev = nullptr;  // mapped [2]: global, status
    uint32_t *ring_cnt = nullptr;      // [2][ring_cnt_n] ring-forwarding chunk counters (zero at export)
    uint64_t ring_cnt_n = 0;
    unsigned long long *peer_stats = nullptr;  // [2] bytes read from peer windows (owners / forwarders)
};

extern Ctx *g_ctx;

void set_error(const char *fmt, ...);
int cuda_fail(cudaError_t e, const char *what);
PtrKind classify(const void *p, int device);
void *pinned_device_alias(const void *p);  // device alias of pinned host memory, else nullptr
int validate_region(const void *out, const void *ref, uint64_t n, int dtype, double abs_tol, double rel_tol,
                    uint64_t max_report, const arc_verify_result_t *res);
int launch_segments(Ctx &c, Seg *segs, uint32_t n_segs, uint32_t acc_lo, uint32_t n_acc, bool finalize);
int wait_results(Ctx &c);
int run_local(Ctx &c, const arc_verify_region_t *regs, size_t R, arc_verify_result_t *results,
              arc_mismatch_t *const *dev_reports, bool d2h_reports, Acc *summaries_out);

// arcv_shard.cu
int shard_init(Ctx &c, const void *nccl_unique_id);
void shard_finalize(Ctx &c);
int shard_compare(Ctx &c, const arc_verify_region_t &r, arc_verify_result_t *result);
int report_target(Ctx &c, arc_verify_result_t *result, uint64_t cap, arc_mismatch_t **dst, bool *host);
void fill_result(const arc_shard_header_t &g, uint64_t max_report, arc_verify_result_t *res);

// arcv_peer.cu
int peer_compare(Ctx &c, const arc_verify_region_t &r, arc_verify_result_t *result);
void peer_finalize(Ctx &c);

}  // namespace arcv
