// arcv_device.cuh -- sm_100a compare-reduce-compact kernel.
//
// One persistent grid streams both arrays of every segment through a
// cp.async.bulk (TMA bulk-copy engine) ring in shared memory, evaluates the
// element predicate of P:199 (sec. III-A; rules 1-5 in include/arc_verify.h),
// reduces the mismatch count and the max abs/rel error, and compacts the first
// max_report mismatches in ascending index order with a single-pass decoupled
// look-back over per-tile mismatch counts.
//
// Block = 1 producer warp (one elected lane issues the bulk copies, tile tickets
// come from a global atomic so look-back always waits on running CTAs) + 8
// consumer warps.  A tile is kTileBytes of EACH array; the tile's elements are
// assigned to consumer threads in 16-byte vectors, vector v = k*256 + thread,
// k = 0..3, so every warp's shared-memory reads are contiguous 512-byte rows.
//
// Exactness: fp32 inputs are widened exactly to fp64 (cvt.f64.f32, compiled with
// -ftz=false so subnormals survive), the margin is __dadd_rn(abs, __dmul_rn(rel,|y|))
// (never contracted), the division for max_rel_err is IEEE div.rn and is only
// evaluated when it can raise the thread's running max (exact filter, DESIGN.md
// sec. 5.3).  Maxima are order-independent, counts are integers, and the report
// order is fixed by the element index, so the result is bit-identical to the
// oracle for any grid, stage count, batching or chunking.
#pragma once
#include <cstdint>
#include <cstring>
#include <type_traits>
#include <cuda_runtime.h>
#include <math_constants.h>

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
constexpr int kMaxInlineSegs = 8;
static_assert(kVecPerThread == 4, "packed-scan layout assumes 4 vectors per thread");

constexpr uint64_t kValMask = (1ull << 46) - 1;     // saturating look-back value
constexpr uint64_t kFlagA = 1ull << 46;             // tile aggregate published
constexpr uint64_t kFlagP = 2ull << 46;             // inclusive prefix published
constexpr int kEpochShift = 48;

// One contiguous piece of one region (a whole region, or one chunk of a region
// streamed from host memory).  96 bytes.
struct Seg {
    const uint8_t *out;
    const uint8_t *ref;
    uint64_t n;             // elements in this segment
    uint64_t tile_begin;    // launch-local index of the segment's first tile
    uint64_t status_begin;  // look-back status slot of the first tile
    uint64_t chain_begin;   // status slot where this region's chain starts
    uint64_t index_base;    // global element index of element 0
    double abs_tol, rel_tol;
    uint64_t max_report;    // report capacity / truncation for the region
    arc_mismatch_t *report; // device pointer, entries [0, max_report)
    uint32_t acc_slot;
    uint32_t dtype;
};

struct Acc {  // per-region accumulators / result slot, 32 bytes
    unsigned long long count;
    unsigned long long max_abs_bits;
    unsigned long long max_rel_bits;
    unsigned long long pad;
};

struct Params {
    const Seg *segs;          // device table, or nullptr -> inline_segs
    uint32_t n_segs;
    uint32_t n_acc;
    uint64_t total_tiles;
    unsigned long long *ticket;
    unsigned long long ticket_base;
    unsigned long long *done;
    unsigned long long done_base;
    uint64_t *status;
    uint64_t epoch_tag;       // epoch << 48
    Acc *acc;
    Acc *result;
    int finalize;
    uint32_t flags;           // bit0: proxy fence before releasing a stage (diagnostic)
    Seg inline_segs[kMaxInlineSegs];
};

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

// ------------------------------------------------------------------ PTX helpers
__device__ __forceinline__ uint32_t smem_u32(const void *p) {
    return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}
__device__ __forceinline__ void mbar_init(uint64_t *bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t *bar) {
    asm volatile("{\n\t.reg .b64 st;\n\tmbarrier.arrive.shared::cta.b64 st, [%0];\n\t}" ::"r"(smem_u32(bar))
                 : "memory");
}
__device__ __forceinline__ void mbar_arrive_expect_tx(uint64_t *bar, uint32_t bytes) {
    asm volatile("{\n\t.reg .b64 st;\n\tmbarrier.arrive.expect_tx.shared::cta.b64 st, [%0], %1;\n\t}" ::"r"(
                     smem_u32(bar)),
                 "r"(bytes)
                 : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t *bar, uint32_t parity) {
    uint32_t done = 0;
    const uint32_t a = smem_u32(bar);
    while (true) {
        asm volatile(
            "{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\tselp.u32 %0, 1, 0, p;\n\t}"
            : "=r"(done)
            : "r"(a), "r"(parity)
            : "memory");
        if (done) break;
    }
}
__device__ __forceinline__ void bulk_g2s(void *dst, const void *src, uint32_t bytes, uint64_t *bar,
                                         uint64_t policy) {
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1], %2, [%3], %4;" ::"r"(
            smem_u32(dst)),
        "l"(src), "r"(bytes), "r"(smem_u32(bar)), "l"(policy)
        : "memory");
}
__device__ __forceinline__ void consumer_bar() {
    asm volatile("bar.sync 1, %0;" ::"n"(kConsumerThreads) : "memory");
}
__device__ __forceinline__ uint64_t ld_relaxed(const uint64_t *p) {
    uint64_t v;
    asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_relaxed(uint64_t *p, uint64_t v) {
    asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}

__device__ __forceinline__ uint64_t warp_sum_u64(uint64_t v) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    return v;
}
__device__ __forceinline__ uint64_t warp_max_u64(uint64_t v) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        const uint64_t w = __shfl_xor_sync(0xffffffffu, v, o);
        v = w > v ? w : v;
    }
    return v;
}
__device__ __forceinline__ double warp_max_f64(double v) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v = fmax(v, __shfl_xor_sync(0xffffffffu, v, o));
    return v;
}

// ------------------------------------------------------------ element predicate
// Float rules 1-5 (arc_verify.h).  Returns true on mismatch; folds d into `ma`
// and r into `rm` (running maxima, NaN-ignoring via fmax).
__device__ __forceinline__ bool eval_f64(double x, double y, double at, double rt, double &ma, double &rm) {
    const double d = fabs(x - y);             // NaN iff an operand is NaN (or Inf - Inf)
    const double ay = fabs(y);
    const double t = __dadd_rn(at, __dmul_rn(rt, ay));
    const bool match = (x == y) | ((x != x) & (y != y)) | ((ay < CUDART_INF) & (d <= t));
    ma = fmax(ma, d);                          // rule 1: x == y -> d = 0 (or NaN for equal Inf: ignored)
    // r > rm is only possible if d >= RN(rm * |y|) (monotone rounding); the
    // negated compare also lets NaN products through (rm = 0, |y| = Inf).
    if ((d > 0.0) & !(d < rm * ay)) {
        const double r = (ay == CUDART_INF) ? CUDART_INF : d / ay;  // rule 4 / rule 5
        rm = fmax(rm, r);
    }
    return !match;
}

template <typename T>
__device__ __forceinline__ uint64_t int_absdiff(T a, T b) {
    if constexpr (sizeof(T) == 8) {
        return a >= b ? (uint64_t)a - (uint64_t)b : (uint64_t)b - (uint64_t)a;
    } else {
        const int64_t d = (int64_t)a - (int64_t)b;
        return (uint64_t)(d < 0 ? -d : d);
    }
}

template <typename T>
__device__ __forceinline__ uint64_t raw_bits(T v) {
    if constexpr (sizeof(T) == 8) {
        uint64_t b;
        memcpy(&b, &v, 8);
        return b;
    } else if constexpr (sizeof(T) == 4) {
        uint32_t b;
        memcpy(&b, &v, 4);
        return b;
    } else {
        return (uint8_t)v;
    }
}

struct ThreadAcc {
    uint64_t count;
    double ma, rm;     // float dtypes
    uint64_t imax;     // integer dtypes
    __device__ void reset() { count = 0; ma = 0.0; rm = 0.0; imax = 0; }
};

// Evaluate this thread's share of one tile; returns the mismatch bit mask
// (bit k*EPV + j <-> tile element (k*256 + ctid)*EPV + j).
template <typename T, bool kFull, bool kAligned>
__device__ __forceinline__ uint64_t eval_tile(const uint8_t *so, const uint8_t *sr, uint32_t off_o, uint32_t off_r,
                                              uint32_t cnt, int ctid, double at, double rt, ThreadAcc &acc) {
    constexpr int EPV = 16 / sizeof(T);
    uint64_t mask = 0;
#pragma unroll
    for (int k = 0; k < kVecPerThread; ++k) {
        const uint32_t v = k * kConsumerThreads + ctid;
        T xo[EPV], xr[EPV];
        if constexpr (kAligned) {
            const uint4 a = reinterpret_cast<const uint4 *>(so)[v];
            const uint4 b = reinterpret_cast<const uint4 *>(sr)[v];
            memcpy(xo, &a, 16);
            memcpy(xr, &b, 16);
        } else {
#pragma unroll
            for (int j = 0; j < EPV; ++j) {
                xo[j] = *reinterpret_cast<const T *>(so + off_o + (v * EPV + j) * sizeof(T));
                xr[j] = *reinterpret_cast<const T *>(sr + off_r + (v * EPV + j) * sizeof(T));
            }
        }
#pragma unroll
        for (int j = 0; j < EPV; ++j) {
            const uint32_t e = v * EPV + j;
            if (kFull || e < cnt) {
                bool mis;
                if constexpr (std::is_floating_point<T>::value) {
                    mis = eval_f64((double)xo[j], (double)xr[j], at, rt, acc.ma, acc.rm);
                } else {
                    const uint64_t m = int_absdiff<T>(xo[j], xr[j]);
                    acc.imax = m > acc.imax ? m : acc.imax;
                    mis = m != 0;
                }
                mask |= (uint64_t)mis << (k * EPV + j);
            }
        }
    }
    return mask;
}

template <typename T>
__device__ __forceinline__ uint64_t eval_tile_dispatch(const uint8_t *so, const uint8_t *sr, const StageInfo &si,
                                                       int ctid, double at, double rt, ThreadAcc &acc) {
    constexpr uint32_t TE = kTileBytes / sizeof(T);
    const bool full = si.count == TE;
    const bool aligned = (si.off_o | si.off_r) == 0;
    if (full) {
        if (aligned) return eval_tile<T, true, true>(so, sr, 0, 0, TE, ctid, at, rt, acc);
        return eval_tile<T, true, false>(so, sr, si.off_o, si.off_r, TE, ctid, at, rt, acc);
    }
    if (aligned) return eval_tile<T, false, true>(so, sr, 0, 0, si.count, ctid, at, rt, acc);
    return eval_tile<T, false, false>(so, sr, si.off_o, si.off_r, si.count, ctid, at, rt, acc);
}

// ------------------------------------------------------------------- look-back
// Executed by one full warp.  Publishes the tile's aggregate, walks back over
// predecessors (32 at a time) until an inclusive prefix is found, publishes the
// tile's inclusive prefix and returns the exclusive prefix (all saturating at
// `sat` = min(max_report, 2^46 - 1)).
__device__ __forceinline__ uint64_t lookback(uint64_t *status, uint64_t slot, uint64_t chain_begin, uint64_t agg,
                                             uint64_t sat, uint64_t tag, int lane) {
    const uint64_t aggs = agg < sat ? agg : sat;
    if (slot == chain_begin) {
        if (lane == 0) st_relaxed(status + slot, tag | kFlagP | aggs);
        return 0;
    }
    if (lane == 0) st_relaxed(status + slot, tag | kFlagA | aggs);
    uint64_t excl = 0;
    int64_t pos = (int64_t)slot - 1;
    const uint64_t epoch = tag >> kEpochShift;
    while (true) {
        const int64_t idx = pos - lane;
        const bool in_chain = idx >= (int64_t)chain_begin;
        uint64_t val = 0;
        uint32_t flag = 2;  // outside the chain: behaves as prefix 0
        uint32_t spins = 0;
        while (true) {
            if (in_chain) {
                const uint64_t w = ld_relaxed(status + idx);
                flag = ((w >> kEpochShift) == epoch) ? (uint32_t)((w >> 46) & 3) : 0u;
                val = w & kValMask;
            }
            const uint32_t pm = __ballot_sync(0xffffffffu, flag == 2);
            const uint32_t xm = __ballot_sync(0xffffffffu, flag == 0);
            const int pl = pm ? __ffs(pm) - 1 : 32;
            const uint32_t rel = pl >= 31 ? 0xffffffffu : ((2u << pl) - 1u);
            if (xm & rel) {
                if (++spins > 4) __nanosleep(64);
                continue;
            }
            const uint64_t v = warp_sum_u64(((rel >> lane) & 1u) ? val : 0ull);
            excl += v;
            excl = excl < sat ? excl : sat;
            if (pl < 32 || excl >= sat) {
                if (lane == 0) {
                    const uint64_t inc = excl + aggs;
                    st_relaxed(status + slot, tag | kFlagP | (inc < sat ? inc : sat));
                }
                return excl;
            }
            break;
        }
        pos -= 32;
    }
}

// ------------------------------------------------------------------ compaction
// Writes this tile's mismatches with global report rank excl + in-tile rank,
// for ranks < max_report.  In-tile order = element index order = (k, ctid, j).
template <typename T>
__device__ __noinline__ void compact_tile(const Seg &g, const StageInfo &si, uint64_t mask, uint64_t excl, int ctid,
                                          uint64_t *s_scan) {
    constexpr int EPV = 16 / sizeof(T);
    constexpr uint64_t kGroup = EPV == 64 ? ~0ull : ((1ull << EPV) - 1ull);
    const int lane = ctid & 31, cw = ctid >> 5;
    uint64_t packed = 0;
#pragma unroll
    for (int k = 0; k < kVecPerThread; ++k)
        packed |= (uint64_t)__popcll(mask & (kGroup << (k * EPV))) << (16 * k);
    uint64_t inc = packed;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const uint64_t y = __shfl_up_sync(0xffffffffu, inc, o);
        if (lane >= o) inc += y;
    }
    if (lane == 31) s_scan[cw] = inc;
    consumer_bar();
    uint64_t wbase = 0, total = 0;
#pragma unroll
    for (int w = 0; w < kConsumerWarps; ++w) {
        const uint64_t x = s_scan[w];
        wbase += (w < cw) ? x : 0ull;
        total += x;
    }
    // no trailing barrier: s_scan is rewritten only after the next tile's two
    // look-back barriers, which every consumer thread passes after this read.
    const uint64_t ex = wbase + inc - packed;
    uint64_t m = mask;
    while (m) {
        const int b = __ffsll((long long)m) - 1;
        m &= m - 1;
        const int k = b / EPV, j = b % EPV;
        uint64_t rank = ((ex >> (16 * k)) & 0xffffull) +
                        (uint64_t)__popcll(mask & (((1ull << j) - 1ull) << (k * EPV)));
        for (int kk = 0; kk < k; ++kk) rank += (total >> (16 * kk)) & 0xffffull;
        const uint64_t gi = excl + rank;
        if (gi < g.max_report) {
            const uint64_t le = si.elem_begin + (uint64_t)((k * kConsumerThreads + ctid) * EPV + j);
            const T *po = reinterpret_cast<const T *>(g.out) + le;
            const T *pr = reinterpret_cast<const T *>(g.ref) + le;
            arc_mismatch_t *dst = g.report + gi;
            dst->index = g.index_base + le;
            dst->out_bits = raw_bits<T>(*po);
            dst->ref_bits = raw_bits<T>(*pr);
        }
    }
}

__device__ __forceinline__ uint32_t find_seg(const Seg *segs, uint32_t n, uint64_t t) {
    uint32_t lo = 0, hi = n;  // last seg with tile_begin <= t
    while (hi - lo > 1) {
        const uint32_t mid = (lo + hi) >> 1;
        if (segs[mid].tile_begin <= t) lo = mid; else hi = mid;
    }
    return lo;
}

// --------------------------------------------------------------------- kernel
template <int S>
__global__ void __launch_bounds__(kThreads, 2) arcv_compare_kernel(const __grid_constant__ Params p) {
    extern __shared__ __align__(128) uint8_t smem[];
    __shared__ __align__(8) uint64_t full_bar[S];
    __shared__ __align__(8) uint64_t empty_bar[S];
    __shared__ StageInfo info[S];
    __shared__ uint64_t s_scan[kConsumerWarps];
    __shared__ uint64_t s_red_u[kConsumerWarps][2];
    __shared__ double s_red_d[kConsumerWarps][2];
    __shared__ uint64_t s_excl;
    __shared__ uint32_t s_agg;
    __shared__ int s_last;

    const Seg *segs = p.segs ? p.segs : p.inline_segs;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;

    if (threadIdx.x == 0) {
        for (int s = 0; s < S; ++s) {
            mbar_init(&full_bar[s], 1);
            mbar_init(&empty_bar[s], kConsumerWarps);
        }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();

    // ------------------------------------------------------------ producer
    if (warp == 0) {
        if (lane == 0) {
            uint64_t policy;
            asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(policy));
            for (uint32_t i = 0;; ++i) {
                const int s = i % S;
                if (i >= (uint32_t)S) mbar_wait(&empty_bar[s], ((i / S) - 1) & 1);
                const uint64_t t = atomicAdd(p.ticket, 1ull) - p.ticket_base;
                if (t >= p.total_tiles) {
                    info[s].tile = ~0ull;
                    mbar_arrive(&full_bar[s]);
                    break;
                }
                const uint32_t sg = find_seg(segs, p.n_segs, t);
                const Seg &g = segs[sg];
                const uint32_t es = elem_size(g.dtype);
                const uint64_t te = kTileBytes / es;
                const uint64_t e0 = (t - g.tile_begin) * te;
                const uint64_t rem = g.n - e0;
                const uint32_t cnt = (uint32_t)(rem < te ? rem : te);
                const uintptr_t bo = reinterpret_cast<uintptr_t>(g.out) + e0 * es;
                const uintptr_t br = reinterpret_cast<uintptr_t>(g.ref) + e0 * es;
                const uintptr_t ao = bo & ~(uintptr_t)15, ar = br & ~(uintptr_t)15;
                const uint32_t nbo = (uint32_t)(((bo + (uint64_t)cnt * es + 15) & ~(uintptr_t)15) - ao);
                const uint32_t nbr = (uint32_t)(((br + (uint64_t)cnt * es + 15) & ~(uintptr_t)15) - ar);
                StageInfo &si = info[s];
                si.tile = t;
                si.elem_begin = e0;
                si.seg = sg;
                si.count = cnt;
                si.off_o = (uint32_t)(bo - ao);
                si.off_r = (uint32_t)(br - ar);
                uint8_t *dst = smem + (size_t)s * kStageBytes;
                mbar_arrive_expect_tx(&full_bar[s], nbo + nbr);
                bulk_g2s(dst, reinterpret_cast<const void *>(ao), nbo, &full_bar[s], policy);
                bulk_g2s(dst + kStageArrayBytes, reinterpret_cast<const void *>(ar), nbr, &full_bar[s], policy);
            }
        }
        return;
    }

    // ------------------------------------------------------------ consumers
    const int ctid = threadIdx.x - 32;
    const int cw = warp - 1;
    ThreadAcc acc;
    acc.reset();
    int cur = -1;
    uint32_t cur_dtype = 0, cur_slot = 0;

    auto flush = [&](uint32_t slot, uint32_t dtype) {
        const bool is_float = dtype == ARC_F32 || dtype == ARC_F64;
        const double mabs = is_float ? acc.ma : __ull2double_rn(acc.imax);
        uint64_t c = warp_sum_u64(acc.count);
        const double wa = warp_max_f64(mabs);
        const double wr = warp_max_f64(acc.rm);
        if (lane == 0) {
            s_red_u[cw][0] = c;
            s_red_d[cw][0] = wa;
            s_red_d[cw][1] = wr;
        }
        consumer_bar();
        if (ctid == 0) {
            uint64_t tc = 0;
            double ta = 0.0, tr = 0.0;
            for (int w = 0; w < kConsumerWarps; ++w) {
                tc += s_red_u[w][0];
                ta = fmax(ta, s_red_d[w][0]);
                tr = fmax(tr, s_red_d[w][1]);
            }
            Acc *a = p.acc + slot;
            if (tc) atomicAdd(&a->count, (unsigned long long)tc);
            if (ta > 0.0) atomicMax(&a->max_abs_bits, (unsigned long long)__double_as_longlong(ta));
            if (tr > 0.0) atomicMax(&a->max_rel_bits, (unsigned long long)__double_as_longlong(tr));
        }
        consumer_bar();
        acc.reset();
    };

    for (uint32_t i = 0;; ++i) {
        const int s = i % S;
        mbar_wait(&full_bar[s], (i / S) & 1);
        const StageInfo si = info[s];
        if (si.tile == ~0ull) break;
        const Seg &g = segs[si.seg];
        if ((int)si.seg != cur) {
            if (cur >= 0 && g.acc_slot != cur_slot) flush(cur_slot, cur_dtype);
            cur = (int)si.seg;
            cur_dtype = g.dtype;
            cur_slot = g.acc_slot;
        }
        const uint8_t *so = smem + (size_t)s * kStageBytes;
        const uint8_t *sr = so + kStageArrayBytes;
        uint64_t mask;
        switch (g.dtype) {
            case ARC_F32: mask = eval_tile_dispatch<float>(so, sr, si, ctid, g.abs_tol, g.rel_tol, acc); break;
            case ARC_F64: mask = eval_tile_dispatch<double>(so, sr, si, ctid, g.abs_tol, g.rel_tol, acc); break;
            case ARC_I32: mask = eval_tile_dispatch<int32_t>(so, sr, si, ctid, 0.0, 0.0, acc); break;
            case ARC_I64: mask = eval_tile_dispatch<int64_t>(so, sr, si, ctid, 0.0, 0.0, acc); break;
            default: mask = eval_tile_dispatch<uint8_t>(so, sr, si, ctid, 0.0, 0.0, acc); break;
        }
        if (p.flags & 1u) asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
        __syncwarp();
        if (lane == 0) mbar_arrive(&empty_bar[s]);  // stage may be refilled now
        const uint32_t cnt = (uint32_t)__popcll(mask);
        acc.count += cnt;

        if (g.max_report == 0) continue;  // count-only: no ordering needed

        const uint32_t wc = __reduce_add_sync(0xffffffffu, cnt);
        if (lane == 0) s_red_u[cw][1] = wc;
        consumer_bar();
        if (cw == 0) {
            uint64_t agg = lane < kConsumerWarps ? s_red_u[lane][1] : 0ull;
            agg = warp_sum_u64(agg);
            const uint64_t sat = g.max_report < kValMask ? g.max_report : kValMask;
            const uint64_t slot = g.status_begin + (si.tile - g.tile_begin);
            const uint64_t excl = lookback(p.status, slot, g.chain_begin, agg, sat, p.epoch_tag, lane);
            if (lane == 0) {
                s_excl = excl;
                s_agg = (uint32_t)agg;
            }
        }
        consumer_bar();
        const uint64_t excl = s_excl;
        const uint32_t agg = s_agg;
        if (agg > 0 && excl < g.max_report) {
            switch (g.dtype) {
                case ARC_F32: compact_tile<float>(g, si, mask, excl, ctid, s_scan); break;
                case ARC_F64: compact_tile<double>(g, si, mask, excl, ctid, s_scan); break;
                case ARC_I32: compact_tile<int32_t>(g, si, mask, excl, ctid, s_scan); break;
                case ARC_I64: compact_tile<int64_t>(g, si, mask, excl, ctid, s_scan); break;
                default: compact_tile<uint8_t>(g, si, mask, excl, ctid, s_scan); break;
            }
        }
        // s_excl / s_agg / s_red_u[.][1] are rewritten only after the next tile's
        // first barrier, which every consumer passes after reading them here.
    }
    if (cur >= 0) flush(cur_slot, cur_dtype);

    if (!p.finalize) return;
    // Last CTA to finish publishes the accumulators and clears them for the next call.
    if (ctid == 0) {
        __threadfence();
        const unsigned long long prev = atomicAdd(p.done, 1ull);
        s_last = (prev - p.done_base) == (unsigned long long)(gridDim.x - 1);
    }
    consumer_bar();
    if (s_last) {
        __threadfence();
        for (uint32_t k = ctid; k < p.n_acc; k += kConsumerThreads) {
            Acc a;
            a.count = __ldcg(&p.acc[k].count);
            a.max_abs_bits = __ldcg(&p.acc[k].max_abs_bits);
            a.max_rel_bits = __ldcg(&p.acc[k].max_rel_bits);
            a.pad = 0;
            p.result[k] = a;
            p.acc[k].count = 0;
            p.acc[k].max_abs_bits = 0;
            p.acc[k].max_rel_bits = 0;
        }
    }
}

}  // namespace arcv
