// arcv_host.cu -- C ABI of include/arc_verify.h: context, workspace, launch
// planning, host-input streaming, result materialisation.
//
// Steps of the hot path: a1 validation + dispatch happens
// here; a2-a4 run in arcv_stream_kernel and a5 in arcv_compact_kernel
// (arcv_device.cuh); a6 (summary and report to the host) and a7 (one grid over
// many regions) are planned here; a8 (cross-GPU merge) lives in arcv_shard.cu.
#include <cuda_runtime.h>

#include <algorithm>
#include <cmath>
#include <cstdarg>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <vector>

#include "arc_verify.h"
#include "arcv_device.cuh"
#include "arcv_internal.h"

namespace arcv {

static char g_err[512] = "";

void set_error(const char *fmt, ...) {
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(g_err, sizeof(g_err), fmt, ap);
    va_end(ap);
}

int cuda_fail(cudaError_t e, const char *what) {
    set_error("%s: %s", what, cudaGetErrorString(e));
    return ARC_E_CUDA;
}

#define CK(call)                                                 \
    do {                                                         \
        cudaError_t e_ = (call);                                 \
        if (e_ != cudaSuccess) return cuda_fail(e_, #call);      \
    } while (0)

Ctx *g_ctx = nullptr;

// ------------------------------------------------------------------ kernels
template <int NSEG>
using KernelFnN = void (*)(ParamsN<NSEG>);
// Variants: (stages, min CTAs per SM).  Stage ring bytes per SM stay within
// the 228 KB shared memory: 3x2 (default), 2x3, 4x1, 6x1.  NSEG: inline
// segments in the parameter block (1 or kMaxInlineSegs).
template <int NSEG>
static KernelFnN<NSEG> stream_kernel_for(int s) {
    switch (s) {
        case 2: return arcv_stream_kernel<2, 3, NSEG>;
        case 4: return arcv_stream_kernel<4, 1, NSEG>;
        case 6: return arcv_stream_kernel<6, 1, NSEG>;
        default: return arcv_stream_kernel<3, 2, NSEG>;
    }
}

// Launch K1 (cooperative when `coop`) and, when `k2`, the separate report
// kernel, with a parameter block of NSEG inline segments.
template <int NSEG>
static cudaError_t launch_k1_k2(const Params &base, const Seg *inl, uint32_t n_inl, uint32_t grid, size_t smem,
                                cudaStream_t st, bool coop, bool k2, uint32_t grid2, bool *pdl, const Params *k2p) {
    ParamsN<NSEG> pn;
    static_cast<Params &>(pn) = base;
    if (n_inl) memcpy(pn.inline_segs, inl, n_inl * sizeof(Seg));
    cudaError_t e;
    if (coop) {
        cudaLaunchConfig_t cfg = {};
        cfg.gridDim = dim3(grid);
        cfg.blockDim = dim3(kThreads);
        cfg.dynamicSmemBytes = smem;
        cfg.stream = st;
        cudaLaunchAttribute at[1];
        at[0].id = cudaLaunchAttributeCooperative;
        at[0].val.cooperative = 1;
        cfg.attrs = at;
        cfg.numAttrs = 1;
        e = cudaLaunchKernelEx(&cfg, stream_kernel_for<NSEG>(g_ctx->stages), pn);
    } else {
        stream_kernel_for<NSEG>(g_ctx->stages)<<<grid, kThreads, smem, st>>>(pn);
        e = cudaGetLastError();
    }
    if (e != cudaSuccess || !k2) return e;
    static_cast<Params &>(pn) = *k2p;
    // cooperative (the group path has a grid barrier) and, unless disabled, a
    // programmatic dependent of K1: its launch overlaps K1's tail
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(grid2);
    cfg.blockDim = dim3(kConsumerThreads);
    cfg.dynamicSmemBytes = kReportSmem;
    cfg.stream = st;
    cudaLaunchAttribute at[2];
    at[0].id = cudaLaunchAttributeCooperative;
    at[0].val.cooperative = 1;
    at[1].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    at[1].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = at;
    cfg.numAttrs = *pdl ? 2 : 1;
    e = cudaLaunchKernelEx(&cfg, arcv_compact_kernel<NSEG>, pn);
    if (e != cudaSuccess && *pdl) {  // PDL refused with a cooperative launch: plain cooperative
        cudaGetLastError();
        *pdl = false;
        cfg.numAttrs = 1;
        e = cudaLaunchKernelEx(&cfg, arcv_compact_kernel<NSEG>, pn);
    }
    return e;
}

static int env_int(const char *name, int dflt) {
    const char *v = getenv(name);
    return v && *v ? atoi(v) : dflt;
}

// ---------------------------------------------------------- device buffers
template <typename T>
static int grow_device(T **p, size_t *cap, size_t need, bool zero, cudaStream_t st) {
    if (need <= *cap) return ARC_OK;
    size_t ncap = std::max(need, *cap * 2);
    if (*p) {
        CK(cudaStreamSynchronize(st));
        CK(cudaFree(*p));
        *p = nullptr;
        *cap = 0;
    }
    cudaError_t e = cudaMalloc(reinterpret_cast<void **>(p), ncap * sizeof(T));
    if (e != cudaSuccess) {
        cudaGetLastError();
        set_error("cudaMalloc(%zu bytes) failed: %s", ncap * sizeof(T), cudaGetErrorString(e));
        return ARC_E_NOMEM;
    }
    if (zero) CK(cudaMemsetAsync(*p, 0, ncap * sizeof(T), st));
    *cap = ncap;
    return ARC_OK;
}

template <typename T>
static int grow_pinned(T **p, size_t *cap, size_t need) {
    if (need <= *cap) return ARC_OK;
    size_t ncap = std::max(need, *cap * 2);
    if (*p) CK(cudaFreeHost(*p));
    *p = nullptr;
    *cap = 0;
    cudaError_t e = cudaMallocHost(reinterpret_cast<void **>(p), ncap * sizeof(T));
    if (e != cudaSuccess) {
        cudaGetLastError();
        set_error("cudaMallocHost(%zu bytes) failed: %s", ncap * sizeof(T), cudaGetErrorString(e));
        return ARC_E_NOMEM;
    }
    *cap = ncap;
    return ARC_OK;
}

PtrKind classify(const void *p, int device) {
    cudaPointerAttributes a;
    cudaError_t e = cudaPointerGetAttributes(&a, p);
    if (e != cudaSuccess) {
        cudaGetLastError();
        return PK_HOST;
    }
    switch (a.type) {
        case cudaMemoryTypeDevice: return a.device == device ? PK_DEVICE : PK_BAD;
        case cudaMemoryTypeManaged: return PK_DEVICE;
        default: return PK_HOST;  // pinned (cudaMemoryTypeHost) or pageable
    }
}

constexpr int kCompactSmem = kReportSmem;

// Pinned host reports with a capacity up to Ctx::direct_max entries are
// written by the kernel over PCIe; larger ones are staged in HBM and copied
// with one bulk D2H (ARCV_DIRECT_MAX overrides the default).
constexpr uint64_t kDirectReportMax = 1 << 16;

// Device alias of page-locked host memory (cudaMallocHost / cudaHostRegister /
// torch pin_memory), or NULL.  Kernels write small results there directly.
void *pinned_device_alias(const void *p) {
    cudaPointerAttributes a;
    if (cudaPointerGetAttributes(&a, p) != cudaSuccess) {
        cudaGetLastError();
        return nullptr;
    }
    return a.type == cudaMemoryTypeHost ? a.devicePointer : nullptr;
}

int validate_region(const void *out, const void *ref, uint64_t n, int dtype, double abs_tol, double rel_tol,
                    uint64_t max_report, const arc_verify_result_t *res) {
    if (!res) { set_error("result is NULL"); return ARC_E_INVAL; }
    if (dtype < ARC_F32 || dtype > ARC_U8) { set_error("unknown dtype %d", dtype); return ARC_E_INVAL; }
    if (!(abs_tol >= 0.0) || !(rel_tol >= 0.0) || std::isinf(abs_tol) || std::isinf(rel_tol)) {
        set_error("tolerances must be finite and >= 0 (abs_tol=%g rel_tol=%g)", abs_tol, rel_tol);
        return ARC_E_INVAL;
    }
    if (n > 0 && (!out || !ref)) { set_error("NULL array with n > 0"); return ARC_E_INVAL; }
    if (max_report > 0 && !res->report) { set_error("report is NULL with max_report > 0"); return ARC_E_INVAL; }
    const uintptr_t es = elem_size((uint32_t)dtype);
    if (n > 0 && (((uintptr_t)out % es) || ((uintptr_t)ref % es))) {
        set_error("array pointer not aligned to the element size");
        return ARC_E_INVAL;
    }
    return ARC_OK;
}

static int validate_check(const arc_verify_check_t *ck) {
    if (!ck) return ARC_OK;
    if (ck->flags & ~(uint32_t)(ARC_CHECK_MIN_VALUE | ARC_CHECK_VALUE_BOUNDS)) {
        set_error("unknown check flags 0x%x", ck->flags);
        return ARC_E_INVAL;
    }
    if (((ck->flags & ARC_CHECK_MIN_VALUE) && std::isnan(ck->min_value)) ||
        ((ck->flags & ARC_CHECK_VALUE_BOUNDS) && (std::isnan(ck->lo) || std::isnan(ck->hi)))) {
        set_error("check parameters must not be NaN");
        return ARC_E_INVAL;
    }
    return ARC_OK;
}

// A float strictly below v (0 when v == 0): the fp32 pre-filter's tolerance
// bounds (arcv_device.cuh eval_f32).
static float lower_f32(double v) {
    if (!(v > 0.0)) return 0.f;
    float f = (float)v;
    if ((double)f > v) f = nextafterf(f, 0.f);
    f = nextafterf(f, 0.f);
    return f > 0.f ? f : 0.f;
}

static uint64_t tiles_of(uint64_t n, uint32_t dtype) {
    const uint64_t te = tile_elems(dtype);
    return (n + te - 1) / te;
}

static Seg make_seg(const void *out, const void *ref, uint64_t n, uint32_t dtype, double at, double rt,
                    uint64_t max_report, arc_mismatch_t *report, uint64_t slot_begin, uint64_t index_base,
                    uint32_t acc_slot, uint32_t flags, const arc_verify_check_t *ck = nullptr) {
    Seg g;
    memset(&g, 0, sizeof(g));
    g.out = static_cast<const uint8_t *>(out);
    g.ref = static_cast<const uint8_t *>(ref);
    g.n = n;
    g.slot_begin = slot_begin;
    g.index_base = index_base;
    g.abs_tol = at;
    g.rel_tol = rt;
    g.max_report = report ? max_report : 0;
    g.report = report;
    g.acc_slot = acc_slot;
    g.dtype = dtype;
    g.flags = flags;
    g.at_rd = lower_f32(at);
    g.rt_rd = lower_f32(rt);
    if (ck && ck->flags) {
        g.cflags = ck->flags;
        g.minv = ck->min_value;
        g.lo = ck->lo;
        g.hi = ck->hi;
    }
    return g;
}

// ------------------------------------------------------------------ launch
// One K1 (its report phase fused, or + K2) over `segs`.  Fills each seg's
// tile_begin / group_begin.  Accumulator slots [acc_lo, acc_lo + n_acc) are
// published to the result slots when `finalize`.
int launch_segments(Ctx &c, Seg *segs, uint32_t n_segs, uint32_t acc_lo, uint32_t n_acc, bool finalize) {
    uint64_t tiles = 0, groups = 0;
    bool need_compact = false;
    for (uint32_t k = 0; k < n_segs; ++k) {
        segs[k].tile_begin = tiles;
        segs[k].group_begin = groups;
        const uint64_t t = tiles_of(segs[k].n, segs[k].dtype);
        tiles += t;
        if (segs[k].max_report) {
            groups += (t + kGroupTiles - 1) / kGroupTiles;
            need_compact = true;
        }
    }
    if (tiles == 0) return ARC_OK;
    if (groups > c.group_cap) {  // two parity halves, zeroed
        size_t cap2 = c.group_cap * 2;
        int st = grow_device(&c.group_cnt, &cap2, std::max<uint64_t>(groups, 1024) * 2, true, c.stream);
        if (st) return st;
        c.group_cap = cap2 / 2;
    }
    int st = ARC_OK;
    Params p;
    memset(&p, 0, sizeof(p));
    for (uint32_t k = 0; k < n_segs; ++k)
        if (segs[k].report && classify(segs[k].report, c.device) != PK_DEVICE) {
            p.report_host = 1;
            segs[k].flags |= kSegReportHost;
        }
    if (n_segs <= (uint32_t)kMaxInlineSegs) {
        p.segs = nullptr;  // inline (copied into the parameter block at launch)
    } else {
        st = grow_device(&c.seg_dev, &c.seg_dev_cap, n_segs, false, c.stream);
        if (st) return st;
        // seg_host may still feed the previous table copy: wait for that copy
        // only (an event after it), not for the whole stream
        if (c.seg_copy_pending) CK(cudaEventSynchronize(c.ev_seg));
        c.seg_copy_pending = false;
        st = grow_pinned(&c.seg_host, &c.seg_host_cap, n_segs);
        if (st) return st;
        memcpy(c.seg_host, segs, n_segs * sizeof(Seg));
        CK(cudaMemcpyAsync(c.seg_dev, c.seg_host, n_segs * sizeof(Seg), cudaMemcpyHostToDevice, c.stream));
        CK(cudaEventRecord(c.ev_seg, c.stream));
        c.seg_copy_pending = true;
        p.segs = c.seg_dev;
    }
    p.n_segs = n_segs;
    p.n_acc = n_acc;
    p.total_tiles = tiles;
    p.ticket = c.counters;
    p.ticket_base = c.ticket_base;
    p.guided = (ARCV_GUIDED && n_segs > 1) ? 1 : 0;
    p.done = c.counters + 1;
    p.done_base = c.done_base;
    p.tile_cnt = c.tile_cnt;
    p.group_cnt = c.group_cnt + (size_t)c.parity * c.group_cap;
    p.group_zero = c.group_cnt + (size_t)(c.parity ^ 1) * c.group_cap;
    p.n_group_zero = c.group_cap;
    p.active = c.active;
    p.active_cnt = c.active_cnt + c.parity;
    p.active_cnt_zero = c.active_cnt + (c.parity ^ 1);
    p.nz_list = c.nz_list;
    p.nz_cnt = c.nz_cnt + c.parity;
    p.nz_cnt_zero = c.nz_cnt + (c.parity ^ 1);
    p.k2 = need_compact ? 1 : 0;
    p.gbar = c.counters + 2;
    p.gbar_base = c.gbar_base;
    p.acc = c.acc + acc_lo;
    p.result = c.result_dev + acc_lo;
    p.finalize = finalize ? 1 : 0;  // the launch publishes the result slots
    p.flags = (uint32_t)c.flags;
    // ARCV_FLAGS bit 3 (diagnostic): stream sync; deferred (peer) calls wake on the exchange kernel
    p.done_flag = ((c.flags & 8) || c.defer_wait) ? nullptr : c.flag_dev;
    // the host waits for the last finalize launch's number (deferred calls wake
    // on the exchange, which carries its own number)
    if (finalize && !c.defer_wait) p.seq = ++c.seq;
    p.mirror = finalize ? c.mirror_next : nullptr;

    const uint64_t max_grid = (uint64_t)c.num_sms * (uint64_t)c.ctas_per_sm;
    const uint32_t grid = (uint32_t)std::min<uint64_t>(tiles, max_grid);
    const size_t smem = (size_t)c.stages * kStageBytes;
    const bool timed = c.timing && c.n_ev < Ctx::kMaxEv;
    // fused: K1 runs the report phase after a grid barrier (cooperative launch)
    const bool fused = need_compact && c.fused;
    p.fused = fused ? 1 : 0;
    // fused exchange (sharded peer call): the shard's final launch runs the
    // exchange in its tail -- cooperative too (its CTAs wait for the peers)
    const bool xf = c.x_next != nullptr && finalize && (!need_compact || fused);
    p.xfused = xf ? 1 : 0;
    if (xf) {
        p.x = *c.x_next;
        p.x.done_base = c.peer_done_base;
    }
    // the separate report kernel (K2) gets the same block with its own bases
    const bool k2 = need_compact && !fused;
    const uint32_t grid2 = (uint32_t)c.k2_grid;
    Params p2;
    if (k2) {
        p2 = p;
        p2.finalize = finalize ? 1 : 0;
        const unsigned long long k1_done = (p.finalize || p.k2) ? grid : 0;
        p2.done_base = c.done_base + k1_done;
    }
    if (timed) CK(cudaEventRecord(c.ev[c.n_ev][0], c.stream));
    const uint32_t n_inl = p.segs ? 0u : n_segs;
    cudaError_t e = n_inl > 1
        ? launch_k1_k2<kMaxInlineSegs>(p, segs, n_inl, grid, smem, c.stream, fused || xf, k2, grid2, &c.pdl, &p2)
        : launch_k1_k2<1>(p, segs, n_inl, grid, smem, c.stream, fused || xf, k2, grid2, &c.pdl, &p2);
    if (e != cudaSuccess) return cuda_fail(e, "arcv_stream_kernel / arcv_compact_kernel launch");
    c.launches += k2 ? 2 : 1;
    if (p.guided) c.ticket_base += tiles;  // runs past the end are given back
    else c.ticket_base += tiles + grid;    // every producer's last ticket fails
    if (xf) {
        c.peer_done_base += grid;  // every K1 CTA counts once on the exchange counter
        c.x_taken = true;
    }
    if (fused) {
        // grid barrier + (finalize) the report phase's completion count
        c.done_base += (uint64_t)grid * (finalize ? 2u : 1u);
        c.gbar_base += grid;
    } else if (p.finalize || p.k2) {
        c.done_base += grid;  // K1 counts its CTAs to find its last one
    }
    if (k2) {
        c.gbar_base += grid2;
        if (finalize) c.done_base += grid2;
    }
    if (timed) {
        CK(cudaEventRecord(c.ev[c.n_ev][1], c.stream));
        c.n_ev++;
    }
    c.parity ^= 1;
    return ARC_OK;
}

// Wait until the last finalize launch has published its results: poll the
// mapped completion word (cheaper to wake on than a stream synchronise), and
// fall back to the stream's status so errors surface and nothing can hang.
int wait_results(Ctx &c) {
    if (c.flags & 8) {
        CK(cudaStreamSynchronize(c.stream));
        return ARC_OK;
    }
    const unsigned long long want = c.seq;
    for (uint64_t it = 1;; ++it) {
        if (__atomic_load_n(c.flag_host, __ATOMIC_ACQUIRE) == want) return ARC_OK;
        if ((it & 255) == 0) {
            cudaError_t e = cudaStreamQuery(c.stream);
            if (e == cudaSuccess) return ARC_OK;  // everything enqueued has completed
            if (e != cudaErrorNotReady) return cuda_fail(e, "kernel execution");
        }
        __builtin_ia32_pause();
    }
}

int collect_timing(Ctx &c) {
    if (c.n_ev) CK(cudaEventSynchronize(c.ev[c.n_ev - 1][1]));
    for (int i = 0; i < c.n_ev; ++i) {
        float ms = 0.f;
        CK(cudaEventElapsedTime(&ms, c.ev[i][0], c.ev[i][1]));
        c.timed_ms += ms;
        c.timed_launches++;
    }
    c.n_ev = 0;
    return ARC_OK;
}

// Prepare per-call workspace sizes.
static int begin_call(Ctx &c, uint64_t tile_slots, uint32_t n_acc) {
    int st = grow_device(&c.tile_cnt, &c.tile_cnt_cap, std::max<uint64_t>(tile_slots, 1), true, c.stream);
    if (st) return st;
    st = grow_device(&c.active, &c.active_cap, 2 * c.tile_cnt_cap, false, c.stream);
    if (st) return st;
    st = grow_device(&c.acc, &c.acc_cap, std::max<uint32_t>(n_acc, 1), true, c.stream);
    if (st) return st;
    // result slots live in mapped pinned host memory: the last CTA writes them
    // over PCIe, so a call needs no D2H copy, only one stream sync.
    if (c.result_host_cap < std::max<uint32_t>(n_acc, 1)) {
        if (c.result_host) {
            CK(cudaStreamSynchronize(c.stream));
            CK(cudaFreeHost(c.result_host));
        }
        c.result_host = nullptr;
        c.result_host_cap = 0;
        const size_t cap = std::max<size_t>(std::max<uint32_t>(n_acc, 1), 64);
        cudaError_t e = cudaHostAlloc(reinterpret_cast<void **>(&c.result_host), cap * sizeof(Acc), cudaHostAllocMapped);
        if (e != cudaSuccess) {
            cudaGetLastError();
            set_error("cudaHostAlloc(result slots) failed: %s", cudaGetErrorString(e));
            return ARC_E_NOMEM;
        }
        CK(cudaHostGetDevicePointer(reinterpret_cast<void **>(&c.result_dev), c.result_host, 0));
        c.result_host_cap = cap;
    }
    return ARC_OK;
}

// Stream one region whose out and/or ref live in host memory through the chunk
// ring: H2D copies on the copy stream overlap the compare of the previous chunk.
static int stream_region(Ctx &c, const arc_verify_region_t &r, bool out_dev, bool ref_dev,
                         arc_mismatch_t *report, uint64_t slot_base, uint32_t acc_slot) {
    const uint32_t dtype = (uint32_t)r.dtype;
    const uint64_t es = elem_size(dtype);
    const uint64_t te = tile_elems(dtype);
    const uint64_t chunk_elems = std::max<uint64_t>(te, (Ctx::kChunkBytes / es) / te * te);
    if (!c.chunk_buf[0][0]) {
        for (int b = 0; b < Ctx::kNBuf; ++b)
            for (int s = 0; s < 2; ++s) {
                cudaError_t e = cudaMalloc(&c.chunk_buf[b][s], Ctx::kChunkBytes);
                if (e != cudaSuccess) {
                    cudaGetLastError();
                    set_error("cudaMalloc(chunk buffer) failed: %s", cudaGetErrorString(e));
                    return ARC_E_NOMEM;
                }
            }
    }
    const uint64_t n = r.n;
    const uint64_t nchunks = (n + chunk_elems - 1) / chunk_elems;
    for (uint64_t ci = 0; ci < nchunks; ++ci) {
        const int b = (int)(ci % Ctx::kNBuf);
        const uint64_t e0 = ci * chunk_elems;
        const uint64_t ne = std::min(chunk_elems, n - e0);
        CK(cudaStreamWaitEvent(c.copy_stream, c.ev_free[b], 0));
        const uint8_t *po = static_cast<const uint8_t *>(r.out) + e0 * es;
        const uint8_t *pr = static_cast<const uint8_t *>(r.ref) + e0 * es;
        if (!out_dev) {
            CK(cudaMemcpyAsync(c.chunk_buf[b][0], po, ne * es, cudaMemcpyHostToDevice, c.copy_stream));
            po = static_cast<const uint8_t *>(c.chunk_buf[b][0]);
        }
        if (!ref_dev) {
            CK(cudaMemcpyAsync(c.chunk_buf[b][1], pr, ne * es, cudaMemcpyHostToDevice, c.copy_stream));
            pr = static_cast<const uint8_t *>(c.chunk_buf[b][1]);
        }
        c.h2d_bytes += (out_dev ? 0 : ne * es) + (ref_dev ? 0 : ne * es);
        CK(cudaEventRecord(c.ev_copy[b], c.copy_stream));
        CK(cudaStreamWaitEvent(c.stream, c.ev_copy[b], 0));
        Seg g = make_seg(po, pr, ne, dtype, r.abs_tol, r.rel_tol, r.max_report, report, slot_base + e0 / te, e0, 0,
                         kSegBaseFromAcc, r.check);
        int st = launch_segments(c, &g, 1, acc_slot, 1, ci + 1 == nchunks);
        if (st) return st;
        CK(cudaEventRecord(c.ev_free[b], c.stream));
    }
    return ARC_OK;
}

// Local (single-GPU) verification of R regions.  Results go to results[k]; a
// region's report goes to its device report pointer, or to the device staging
// buffer and then to host memory.  When `dev_reports` is non-NULL the caller
// supplies the device report target per region instead (sharded packets).
int run_local(Ctx &c, const arc_verify_region_t *regs, size_t R, arc_verify_result_t *results,
              arc_mismatch_t *const *dev_reports, bool d2h_reports, Acc *summaries_out) {
    struct Plan {
        bool out_dev, ref_dev, stream;
        arc_mismatch_t *dreport;  // device target
        arc_mismatch_t *alias;    // device alias of a pinned host report (sparse: written directly)
        bool host_report;
        bool pageable;            // host report in pageable memory: sparse entries land in the
                                  // library's pinned staging (pin_off), then one host memcpy
        uint64_t stage_off, pin_off;
        uint64_t tiles, slot_base;
    };
    std::vector<Plan> plan(R);
    uint64_t tile_slots = 0, stage_entries = 0, pin_entries = 0;
    for (size_t k = 0; k < R; ++k) {
        const arc_verify_region_t &r = regs[k];
        int st = validate_region(r.out, r.ref, r.n, r.dtype, r.abs_tol, r.rel_tol, r.max_report, &results[k]);
        if (st) return st;
        st = validate_check(r.check);
        if (st) return st;
        Plan &pl = plan[k];
        pl.out_dev = pl.ref_dev = true;
        if (r.n > 0) {
            const PtrKind ko = classify(r.out, c.device), kr = classify(r.ref, c.device);
            if (ko == PK_BAD || kr == PK_BAD) {
                set_error("region %zu: device pointer belongs to another device", k);
                return ARC_E_INVAL;
            }
            pl.out_dev = ko == PK_DEVICE;
            pl.ref_dev = kr == PK_DEVICE;
        }
        pl.stream = !(pl.out_dev && pl.ref_dev);
        pl.tiles = tiles_of(r.n, (uint32_t)r.dtype);
        pl.slot_base = tile_slots;
        tile_slots += pl.tiles;
        const uint64_t cap = std::min<uint64_t>(r.max_report, r.n);
        pl.host_report = false;
        pl.pageable = false;
        pl.dreport = nullptr;
        pl.alias = nullptr;
        if (cap > 0) {
            if (dev_reports) {
                pl.dreport = dev_reports[k];
            } else if (classify(results[k].report, c.device) == PK_DEVICE) {
                pl.dreport = results[k].report;
            } else if (void *alias = cap <= c.direct_max ? pinned_device_alias(results[k].report) : nullptr) {
                pl.dreport = static_cast<arc_mismatch_t *>(alias);  // small pinned report: written over PCIe by the report phase
            } else {
                pl.host_report = true;
                pl.stage_off = stage_entries;
                stage_entries += cap;
                if (!pl.stream) {
                    pl.alias = static_cast<arc_mismatch_t *>(pinned_device_alias(results[k].report));
                    if (!pl.alias) {  // pageable: the sparse case goes through pinned staging
                        pl.pageable = true;
                        pl.pin_off = pin_entries;
                        pin_entries += std::min<uint64_t>(cap, kDirectDyn);
                    }
                }
            }
        }
    }
    int st = begin_call(c, tile_slots, (uint32_t)R);
    if (st) return st;
    if (stage_entries) {
        st = grow_device(&c.report_stage, &c.report_stage_cap, stage_entries, false, c.stream);
        if (st) return st;
    }
    if (pin_entries > c.report_pin_cap) {  // mapped pinned staging for sparse pageable reports
        if (c.report_pin) {
            CK(cudaStreamSynchronize(c.stream));
            CK(cudaFreeHost(c.report_pin));
        }
        c.report_pin = nullptr;
        c.report_pin_cap = 0;
        const size_t cap = std::max<size_t>(pin_entries, 2 * kDirectDyn);
        cudaError_t e = cudaHostAlloc(reinterpret_cast<void **>(&c.report_pin), cap * sizeof(arc_mismatch_t),
                                      cudaHostAllocMapped);
        if (e != cudaSuccess) {
            cudaGetLastError();
            set_error("cudaHostAlloc(report staging) failed: %s", cudaGetErrorString(e));
            return ARC_E_NOMEM;
        }
        CK(cudaHostGetDevicePointer(reinterpret_cast<void **>(&c.report_pin_dev), c.report_pin, 0));
        c.report_pin_cap = cap;
    }
    for (size_t k = 0; k < R; ++k)
        if (plan[k].pageable) plan[k].alias = c.report_pin_dev + plan[k].pin_off;
    for (size_t k = 0; k < R; ++k)
        if (plan[k].host_report) plan[k].dreport = c.report_stage + plan[k].stage_off;

    // accumulator slots: device-resident regions occupy [0, D) in region order,
    // streamed regions follow (each published by its own last chunk).
    std::vector<uint32_t> slot_of(R, 0);
    std::vector<Seg> segs;
    uint32_t next_slot = 0;
    for (size_t k = 0; k < R; ++k) {
        const arc_verify_region_t &r = regs[k];
        if (plan[k].stream || r.n == 0) continue;
        slot_of[k] = next_slot;
        segs.push_back(make_seg(r.out, r.ref, r.n, (uint32_t)r.dtype, r.abs_tol, r.rel_tol, r.max_report,
                                plan[k].dreport, plan[k].slot_base, 0, next_slot, 0, r.check));
        segs.back().report_alias = plan[k].alias;
        next_slot++;
    }
    const uint32_t n_dev_slots = next_slot;
    for (size_t k = 0; k < R; ++k)
        if (plan[k].stream && regs[k].n > 0) slot_of[k] = next_slot++;

    if (!segs.empty()) {  // one grid over every device-resident region (a7)
        st = launch_segments(c, segs.data(), (uint32_t)segs.size(), 0, n_dev_slots, true);
        if (st) return st;
    }
    for (size_t k = 0; k < R; ++k) {
        if (!plan[k].stream || regs[k].n == 0) continue;
        st = stream_region(c, regs[k], plan[k].out_dev, plan[k].ref_dev, plan[k].dreport, plan[k].slot_base,
                           slot_of[k]);
        if (st) return st;
    }
    if (c.defer_wait) return ARC_OK;  // the peer-exchange kernel reads the mirror
    const uint32_t n_slots = next_slot;
    if (n_slots) {  // result slots are mapped host memory
        st = wait_results(c);
        if (st) return st;
    }
    if (c.timing && c.n_ev > Ctx::kMaxEv - 4) {  // read the event ring lazily: no per-call sync
        st = collect_timing(c);
        if (st) return st;
    }
    for (size_t k = 0; k < R; ++k) {
        const arc_verify_region_t &r = regs[k];
        Acc a;
        memset(&a, 0, sizeof(a));
        if (r.n > 0) a = c.result_host[slot_of[k]];
        if (summaries_out) summaries_out[k] = a;
        arc_verify_result_t &o = results[k];
        o.n = r.n;
        o.n_mismatch = a.count;
        double ma, mr;
        memcpy(&ma, &a.max_abs_bits, 8);
        memcpy(&mr, &a.max_rel_bits, 8);
        o.max_abs_err = ma;
        o.max_rel_err = mr;
        o.n_reported = std::min<uint64_t>(a.count, r.max_report);
    }
    if (d2h_reports) {
        bool any = false;
        for (size_t k = 0; k < R; ++k) {
            if (!plan[k].host_report || results[k].n_reported == 0) continue;
            if (plan[k].alias && results[k].n_mismatch <= kDirectDyn) {  // the kernel wrote it directly
                if (plan[k].pageable)
                    memcpy(results[k].report, c.report_pin + plan[k].pin_off,
                           results[k].n_reported * sizeof(arc_mismatch_t));
                continue;
            }
            CK(cudaMemcpyAsync(results[k].report, plan[k].dreport, results[k].n_reported * sizeof(arc_mismatch_t),
                               cudaMemcpyDeviceToHost, c.stream));
            any = true;
        }
        if (any) CK(cudaStreamSynchronize(c.stream));
    }
    return ARC_OK;
}

}  // namespace arcv

using namespace arcv;

// ====================================================================== C ABI
extern "C" {

uint32_t arc_verify_version(void) { return (1u << 16) | 1u; }

const char *arc_verify_strerror(int status) {
    switch (status) {
        case ARC_OK: return "ok";
        case ARC_E_INVAL: return "invalid argument";
        case ARC_E_NOINIT: return "arc_verify_init has not been called";
        case ARC_E_CUDA: return "CUDA runtime error";
        case ARC_E_NCCL: return "NCCL error";
        case ARC_E_NOMEM: return "out of memory";
        case ARC_E_UNSUPPORTED: return "unsupported request";
        default: return "unknown status";
    }
}

const char *arc_verify_last_error(void) { return g_err; }

int arc_verify_init(const arc_verify_opts_t *opts) {
    if (g_ctx) { set_error("already initialised"); return ARC_E_INVAL; }
    arc_verify_opts_t o;
    memset(&o, 0, sizeof(o));
    o.nranks = 1;
    if (opts) o = *opts;
    if (o.nranks < 1 || o.rank < 0 || o.rank >= o.nranks) { set_error("bad rank/nranks"); return ARC_E_INVAL; }
    // nranks > 1 without an NCCL id: peer-memory exchange only (arc_verify_peer_*
    // must be called before the first collective compare).  An NCCL id selects
    // the collective path even for one rank (a 1-rank communicator), which lets
    // a single GPU exercise it end to end.
    int ndev = 0;
    cudaError_t e = cudaGetDeviceCount(&ndev);
    if (e != cudaSuccess) { cudaGetLastError(); return cuda_fail(e, "cudaGetDeviceCount"); }
    if (o.device < 0 || o.device >= ndev) { set_error("bad device %d (of %d)", o.device, ndev); return ARC_E_INVAL; }
    CK(cudaSetDevice(o.device));
    cudaDeviceProp prop;
    CK(cudaGetDeviceProperties(&prop, o.device));
    if (prop.major < 10) {
        set_error("device %d is sm_%d%d; this build targets sm_100a", o.device, prop.major, prop.minor);
        return ARC_E_UNSUPPORTED;
    }
    Ctx *c = new Ctx();
    c->device = o.device;
    c->rank = o.rank;
    c->nranks = o.nranks;
    c->num_sms = prop.multiProcessorCount;
    if (o.stream) {
        c->stream = static_cast<cudaStream_t>(o.stream);
        c->own_stream = false;
    } else {
        CK(cudaStreamCreateWithFlags(&c->stream, cudaStreamNonBlocking));
        c->own_stream = true;
    }
    CK(cudaStreamCreateWithFlags(&c->copy_stream, cudaStreamNonBlocking));
    for (int b = 0; b < Ctx::kNBuf; ++b) {
        CK(cudaEventCreateWithFlags(&c->ev_copy[b], cudaEventDisableTiming));
        CK(cudaEventCreateWithFlags(&c->ev_free[b], cudaEventDisableTiming));
    }
    CK(cudaEventCreateWithFlags(&c->ev_seg, cudaEventDisableTiming));
    for (int i = 0; i < Ctx::kMaxEv; ++i) {
        CK(cudaEventCreate(&c->ev[i][0]));
        CK(cudaEventCreate(&c->ev[i][1]));
    }
    c->flags = env_int("ARCV_FLAGS", 0);
    c->pdl = env_int("ARCV_PDL", 1) != 0;
    {
        const char *v = getenv("ARCV_DIRECT_MAX");
        c->direct_max = (v && *v) ? strtoull(v, nullptr, 0) : kDirectReportMax;
    }
    c->stages = env_int("ARCV_STAGES", 3);
    if (c->stages != 2 && c->stages != 3 && c->stages != 4 && c->stages != 6) c->stages = 3;
    const size_t smem = (size_t)c->stages * kStageBytes;
    KernelFnN<kMaxInlineSegs> kf = stream_kernel_for<kMaxInlineSegs>(c->stages);
    CK(cudaFuncSetAttribute(kf, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    CK(cudaFuncSetAttribute(stream_kernel_for<1>(c->stages), cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    CK(cudaFuncSetAttribute(arcv_compact_kernel<kMaxInlineSegs>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                            kCompactSmem));
    CK(cudaFuncSetAttribute(arcv_compact_kernel<1>, cudaFuncAttributeMaxDynamicSharedMemorySize, kCompactSmem));
    int occ = 0;
    CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, kf, kThreads, smem));
    if (occ < 1) { set_error("kernel does not fit on an SM (smem %zu)", smem); return ARC_E_UNSUPPORTED; }
    // K2: as many co-resident CTAs as fit (cooperative launch), so the re-read
    // tiles of a sparse report are all in flight in one wave
    int occ2 = 0;
    CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ2, arcv_compact_kernel<kMaxInlineSegs>, kConsumerThreads,
                                                     kCompactSmem));
    const int k2cap = env_int("ARCV_K2_PER_SM", 2);
    c->k2_grid = c->num_sms * std::max(1, std::min(occ2, k2cap > 0 ? k2cap : 1));
    const int cap = env_int("ARCV_CTAS_PER_SM", 0);
    c->ctas_per_sm = cap > 0 ? std::min(cap, occ) : occ;
    // the report phase runs in K1's tail when its stage memory holds the
    // report phase's (>= 3 stages); ARCV_FUSED=0 forces the separate K2
    c->fused = env_int("ARCV_FUSED", 1) != 0 && smem >= (size_t)kReportSmem;
    // the exchange in K1's tail needs its scratch in the stage memory
    c->fused_exchange = env_int("ARCV_FUSED_EXCHANGE", 1) != 0 && smem >= sizeof(ExShared);
    if (env_int("ARCV_VERBOSE", 0)) {
        cudaFuncAttributes fa;
        CK(cudaFuncGetAttributes(&fa, kf));
        fprintf(stderr, "[arcv] sms=%d stages=%d ctas/sm=%d (occupancy %d) k2_grid=%d fused=%d regs=%d static_smem=%zu dyn_smem=%zu local=%zu\n",
                c->num_sms, c->stages, c->ctas_per_sm, occ, c->k2_grid, (int)c->fused, fa.numRegs, fa.sharedSizeBytes, smem, fa.localSizeBytes);
    }
    // counters: [0] tile tickets, [1] finished CTAs, [2] report-phase grid barrier,
    // [3] 2 x u32 active-list lengths, [4] 2 x u32 pool lengths (by parity),
    // [5] peer-exchange finished blocks
    e = cudaMalloc(&c->counters, 8 * sizeof(unsigned long long));
    if (e != cudaSuccess) { cudaGetLastError(); set_error("cudaMalloc counters"); return ARC_E_NOMEM; }
    CK(cudaMemsetAsync(c->counters, 0, 8 * sizeof(unsigned long long), c->stream));
    e = cudaHostAlloc(reinterpret_cast<void **>(&c->flag_host), 64, cudaHostAllocMapped);
    if (e != cudaSuccess) { cudaGetLastError(); set_error("cudaHostAlloc(flag)"); return ARC_E_NOMEM; }
    c->flag_host[0] = 0;
    CK(cudaHostGetDevicePointer(reinterpret_cast<void **>(&c->flag_dev), c->flag_host, 0));
    c->active_cnt = reinterpret_cast<uint32_t *>(c->counters + 3);
    c->nz_cnt = reinterpret_cast<uint32_t *>(c->counters + 4);

    e = cudaMalloc(&c->nz_list, 2 * kPoolCap * sizeof(uint64_t));
    if (e != cudaSuccess) { cudaGetLastError(); set_error("cudaMalloc pool list"); return ARC_E_NOMEM; }
    CK(cudaStreamSynchronize(c->stream));
    g_ctx = c;
    c->sharded = o.nccl_unique_id != nullptr || o.nranks > 1;
    if (o.nccl_unique_id) {
        int st = shard_init(*c, o.nccl_unique_id);
        if (st) {
            arc_verify_finalize();
            return st;
        }
    }
    return ARC_OK;
}

int arc_verify_finalize(void) {
    if (!g_ctx) return ARC_E_NOINIT;
    Ctx *c = g_ctx;
    cudaStreamSynchronize(c->stream);
    peer_finalize(*c);
    shard_finalize(*c);
    cudaFree(c->counters);
    cudaFree(c->tile_cnt);
    cudaFree(c->active);
    cudaFree(c->nz_list);
    cudaFree(c->group_cnt);
    cudaFree(c->acc);
    cudaFree(c->seg_dev);
    cudaFree(c->report_stage);
    cudaFree(c->packet);
    cudaFree(c->gathered);
    if (c->result_host) cudaFreeHost(c->result_host);  // result_dev is its device alias
    if (c->flag_host) cudaFreeHost(c->flag_host);
    if (c->seg_host) cudaFreeHost(c->seg_host);
    if (c->report_pin) cudaFreeHost(c->report_pin);  // report_pin_dev is its device alias
    if (c->hdr_host) cudaFreeHost(c->hdr_host);
    if (c->ev_seg) cudaEventDestroy(c->ev_seg);
    for (int b = 0; b < Ctx::kNBuf; ++b) {
        cudaFree(c->chunk_buf[b][0]);
        cudaFree(c->chunk_buf[b][1]);
        cudaEventDestroy(c->ev_copy[b]);
        cudaEventDestroy(c->ev_free[b]);
    }
    for (int i = 0; i < Ctx::kMaxEv; ++i) {
        cudaEventDestroy(c->ev[i][0]);
        cudaEventDestroy(c->ev[i][1]);
    }
    cudaStreamDestroy(c->copy_stream);
    if (c->own_stream) cudaStreamDestroy(c->stream);
    delete c;
    g_ctx = nullptr;
    return ARC_OK;
}

int arc_verify_set_stream(void *stream) {
    if (!g_ctx) return ARC_E_NOINIT;
    Ctx &c = *g_ctx;
    if (!stream) { set_error("stream is NULL"); return ARC_E_INVAL; }
    CK(cudaStreamSynchronize(c.stream));
    if (c.own_stream) CK(cudaStreamDestroy(c.stream));
    c.stream = static_cast<cudaStream_t>(stream);
    c.own_stream = false;
    return ARC_OK;
}

int arc_verify_set_timing(int enable) {
    if (!g_ctx) return ARC_E_NOINIT;
    g_ctx->timing = enable != 0;
    return ARC_OK;
}

uint64_t arc_verify_launch_count(void) { return g_ctx ? g_ctx->launches : 0; }

int arc_verify_kernel_stats(uint64_t *launches, double *total_ms, int reset) {
    if (!g_ctx) return ARC_E_NOINIT;
    int st = collect_timing(*g_ctx);
    if (st) return st;
    if (launches) *launches = g_ctx->timed_launches;
    if (total_ms) *total_ms = g_ctx->timed_ms;
    if (reset) {
        g_ctx->timed_launches = 0;
        g_ctx->timed_ms = 0.0;
    }
    return ARC_OK;
}

int arc_verify_compare(const void *out, const void *ref, uint64_t n, arc_dtype_t dtype, double abs_tol,
                       double rel_tol, uint64_t max_report, arc_verify_result_t *result) {
    if (!g_ctx) return ARC_E_NOINIT;
    arc_verify_region_t r;
    r.out = out;
    r.ref = ref;
    r.n = n;
    r.dtype = dtype;
    r.abs_tol = abs_tol;
    r.rel_tol = rel_tol;
    r.max_report = max_report;
    r.name = nullptr;
    r.check = nullptr;
    if (g_ctx->sharded) return shard_compare(*g_ctx, r, result);
    return run_local(*g_ctx, &r, 1, result, nullptr, true, nullptr);
}

int arc_verify_compare_ex(const void *out, const void *ref, uint64_t n, arc_dtype_t dtype, double abs_tol,
                          double rel_tol, uint64_t max_report, const arc_verify_check_t *check,
                          arc_verify_result_t *result) {
    if (!g_ctx) return ARC_E_NOINIT;
    arc_verify_region_t r;
    r.out = out;
    r.ref = ref;
    r.n = n;
    r.dtype = dtype;
    r.abs_tol = abs_tol;
    r.rel_tol = rel_tol;
    r.max_report = max_report;
    r.name = nullptr;
    r.check = (check && check->flags) ? check : nullptr;
    if (g_ctx->sharded) return shard_compare(*g_ctx, r, result);
    return run_local(*g_ctx, &r, 1, result, nullptr, true, nullptr);
}

// Diagnostic (A/B builds with -DARCV_TRACE=1 only): copy the per-CTA phase
// stamps of the last traced launch pair, [2][1024][12] u64, into `out`.
extern "C" int arc_verify_debug_trace(unsigned long long *out) {
#if defined(ARCV_TRACE) && ARCV_TRACE
    if (!g_ctx) return ARC_E_NOINIT;
    CK(cudaStreamSynchronize(g_ctx->stream));
    CK(cudaMemcpyFromSymbol(out, arcv::g_trace, sizeof(arcv::g_trace)));
    std::vector<unsigned long long> zero(sizeof(arcv::g_trace) / 8, 0ull);
    CK(cudaMemcpyToSymbol(arcv::g_trace, zero.data(), sizeof(arcv::g_trace)));
    return ARC_OK;
#else
    (void)out;
    set_error("built without ARCV_TRACE");
    return ARC_E_UNSUPPORTED;
#endif
}

int arc_verify_probe_read(const void *a, const void *b, uint64_t bytes, int iters, double *gbs) {
    if (!g_ctx) return ARC_E_NOINIT;
    Ctx &c = *g_ctx;
    if (!a || !b || !gbs || iters < 1 || bytes == 0 || classify(a, c.device) != PK_DEVICE ||
        classify(b, c.device) != PK_DEVICE) {
        set_error("probe: device buffers, bytes > 0, iters >= 1 required");
        return ARC_E_INVAL;
    }
    int st = begin_call(c, tiles_of(bytes, ARC_U8), 1);
    if (st) return st;
    const int saved = c.flags;
    const bool saved_t = c.timing;
    c.flags |= (int)kFlagProbe;
    c.timing = false;
    cudaEvent_t e0, e1;
    CK(cudaEventCreate(&e0));
    CK(cudaEventCreate(&e1));
    Seg g = make_seg(a, b, bytes, ARC_U8, 0.0, 0.0, 0, nullptr, 0, 0, 0, 0);
    st = launch_segments(c, &g, 1, 0, 1, true);  // warm-up
    CK(cudaEventRecord(e0, c.stream));
    for (int i = 0; i < iters && !st; ++i) st = launch_segments(c, &g, 1, 0, 1, true);
    CK(cudaEventRecord(e1, c.stream));
    CK(cudaEventSynchronize(e1));
    float ms = 0.f;
    CK(cudaEventElapsedTime(&ms, e0, e1));
    cudaEventDestroy(e0);
    cudaEventDestroy(e1);
    c.flags = saved;
    c.timing = saved_t;
    if (st) return st;
    *gbs = 2.0 * (double)bytes * iters / (ms * 1e-3) / 1e9;
    return ARC_OK;
}

int arc_verify_batch(const arc_verify_region_t *regions, size_t n_regions, arc_verify_result_t *results) {
    if (!g_ctx) return ARC_E_NOINIT;
    if (n_regions == 0) return ARC_OK;
    if (!regions || !results) { set_error("regions/results is NULL"); return ARC_E_INVAL; }
    return run_local(*g_ctx, regions, n_regions, results, nullptr, true, nullptr);
}

}  // extern "C"
