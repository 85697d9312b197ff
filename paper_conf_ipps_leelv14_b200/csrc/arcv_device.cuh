// arcv_device.cuh -- sm_100a kernels of the kernel-verification comparison.
//
// One kernel per verification call:
//
//  K1 arcv_stream_kernel  -- a2-a4 (+ the counting half of a5).  A persistent
//     grid streams both arrays of every segment through a cp.async.bulk (TMA
//     bulk-copy engine) ring in shared memory, evaluates the element predicate
//     of P:199 (sec. III-A; rules 1-5 in include/arc_verify.h), and reduces the
//     mismatch count and the max abs/rel error.  For regions that want a report
//     it also records per-tile and per-group (256 tiles) mismatch counts with
//     warp-level atomics -- no block barrier, no inter-CTA waiting in the
//     streaming loop.
//  report_phase -- a5, run by K1's consumer warps after a grid barrier when a
//     region wants a report (K1 is then a cooperative launch), or as its own
//     kernel K2 arcv_compact_kernel (fewer than 3 stages, or ARCV_FUSED=0).
//     Scans the group and tile counts (tiny), and re-reads ONLY the tiles whose
//     mismatches fall among the first max_report (exclusive prefix <
//     max_report), writing their entries in ascending index order.  Sparse
//     mismatches cost one extra tile read each; dense ones stop at max_report.
//     The last CTA to finish publishes the per-region summary.
//
// Block of K1 = 1 producer warp (one lane issues bulk copies; tile tickets come
// from a global atomic so the grid is load-balanced) + 8 consumer warps.  A tile
// is kTileBytes of EACH array; its elements are assigned to consumer threads in
// 16-byte vectors, vector v = k*256 + thread, k = 0..3, so each warp's shared
// memory reads are contiguous 512-byte rows.
//
// Exactness: float decisions are made in IEEE fp64 (cvt.f64.f32 with -ftz=false,
// __dadd_rn(abs, __dmul_rn(rel,|y|)), never contracted, IEEE div.rn).  For fp32
// inputs an fp32 pre-filter skips the fp64 work only when the outcome is PROVEN
// identical (match certain, no maximum can change).  Maxima
// are order-independent, counts are integers and the report order is fixed by
// the element index, so results are bit-identical to the oracle for any grid,
// stage count, batching or chunking.
#pragma once
#include <cstdint>
#include <cstring>
#include <type_traits>
#include <cuda_runtime.h>
#include <math_constants.h>

#include "arc_verify.h"
#include "arcv_exchange.cuh"
#include "arcv_types.h"

namespace arcv {

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

// Release/acquire fences for the message-passing patterns of this file (last
// CTA publishes; report entries before a completion word; grid barrier).  None
// of them needs the single total order of fence.sc (what __threadfence() and
// __threadfence_system() emit: MEMBAR.SC.GPU / MEMBAR.SC.SYS); fence.acq_rel
// (MEMBAR.ALL.*) gives the same release and acquire patterns, cheaper.
// -DARCV_FENCE_SC=1 restores the SC fences (A/B builds).
__device__ __forceinline__ void fence_gpu() {
#if defined(ARCV_FENCE_SC) && ARCV_FENCE_SC
    __threadfence();
#else
    asm volatile("fence.acq_rel.gpu;" ::: "memory");
#endif
}
__device__ __forceinline__ void fence_sys() {
#if defined(ARCV_FENCE_SC) && ARCV_FENCE_SC
    __threadfence_system();
#else
    asm volatile("fence.acq_rel.sys;" ::: "memory");
#endif
}

// Diagnostic phase trace (A/B builds only, -DARCV_TRACE=1): %globaltimer stamps
// per CTA, read by arc_verify_debug_trace.  Compiled out otherwise.
#if defined(ARCV_TRACE) && ARCV_TRACE
constexpr int kTraceCtas = 1024, kTracePts = 32, kTraceRows = 3;
// [row][cta][point]: row 0 K1, row 1 report phase, row 2 region switches
// (point 2 seg: switched into segment seg, 2 seg + 1: its first tile evaluated; seg < 16)
__device__ unsigned long long g_trace[kTraceRows][kTraceCtas][kTracePts];
// Host side, one per module: merge (element-wise max) this module's stamps into
// `out` and clear them; the launch that ran stamped only its own module.
#define ARCV_DEFINE_TRACE_COPY(name)                                                                  \
    int name(unsigned long long *out, size_t bytes) {                                                 \
        if (bytes < sizeof(g_trace)) return -1;                                                       \
        const size_t n = sizeof(g_trace) / 8;                                                         \
        unsigned long long *tmp = new unsigned long long[n]();                                        \
        int rc = cudaMemcpyFromSymbol(tmp, g_trace, sizeof(g_trace)) == cudaSuccess ? 0 : -1;         \
        for (size_t i = 0; rc == 0 && i < n; ++i) out[i] = tmp[i] > out[i] ? tmp[i] : out[i];         \
        for (size_t i = 0; i < n; ++i) tmp[i] = 0ull;                                                 \
        if (rc == 0 && cudaMemcpyToSymbol(g_trace, tmp, sizeof(g_trace)) != cudaSuccess) rc = -1;     \
        delete[] tmp;                                                                                 \
        return rc;                                                                                    \
    }
#define ARCV_STAMP(k, pt)                                                                      \
    do {                                                                                       \
        unsigned long long t_;                                                                 \
        asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t_));                               \
        if (blockIdx.x < (unsigned)kTraceCtas) g_trace[k][blockIdx.x][pt] = t_;                \
    } while (0)
#else
#define ARCV_STAMP(k, pt) do {} while (0)
#define ARCV_DEFINE_TRACE_COPY(name)                           \
    int name(unsigned long long *out, size_t bytes) {          \
        (void)out;                                             \
        (void)bytes;                                           \
        return -1;                                             \
    }
#endif

__device__ __forceinline__ uint64_t warp_sum_u64(uint64_t v) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    return v;
}
__device__ __forceinline__ double warp_max_f64(double v) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v = fmax(v, __shfl_xor_sync(0xffffffffu, v, o));
    return v;
}

#define ARCV_PRAGMA_(x) _Pragma(#x)
#define ARCV_UNROLL_(n) ARCV_PRAGMA_(unroll n)
#define ARCV_UNROLL(n) ARCV_UNROLL_(n)
// Code-size knobs (A/B builds): unroll factors of the per-tile vector loop
// (default: all kVecPerThread = 4 vectors) and of the seeding scan (default:
// all elements).  Smaller code = fewer cold instruction lines on the first
// tile of a region (profiles/r02i_stall_summary.txt).
// Per-tile report bookkeeping by the producer lane when a stage comes back
// empty (1), or by the consumer warp that finishes a tile last (0).
#ifndef ARCV_PRODUCER_BOOKKEEP
#define ARCV_PRODUCER_BOOKKEEP 1
#endif
#ifndef ARCV_EVAL_UNROLL
#define ARCV_EVAL_UNROLL 4
#endif
#ifndef ARCV_SEED_UNROLL
#define ARCV_SEED_UNROLL 64
#endif

// ------------------------------------------------------------ element predicate
struct ThreadAcc {
    uint64_t count;
    double ma, rm;     // float dtypes: running max of d and r (fp64, exact)
    uint64_t imax;     // integer dtypes: running max |a - b|
    bool seeded;       // float filter bounds seeded for this region
    __device__ void reset() {
        count = 0; ma = 0.0; rm = 0.0; imax = 0; seeded = false;
    }
};

// The fields of the current segment that the per-tile path needs, cached in
// registers (the Seg table lives in param / global space: generic loads).
struct SegHot {
    double (*seed_sh)[2];  // [kConsumerWarps][2] shared scratch: block-wide seeding
    double abs_tol, rel_tol;
    uint64_t max_report, tile_begin, slot_begin, group_begin;
    float at_rd, rt_rd;
    uint32_t dtype, acc_slot, cflags;
    double minv, lo, hi;
    __device__ __forceinline__ void load(const Seg &g) {
        abs_tol = g.abs_tol; rel_tol = g.rel_tol; max_report = g.max_report;
        tile_begin = g.tile_begin; slot_begin = g.slot_begin; group_begin = g.group_begin;
        at_rd = g.at_rd; rt_rd = g.rt_rd; dtype = g.dtype; acc_slot = g.acc_slot;
        cflags = g.cflags; minv = g.minv; lo = g.lo; hi = g.hi;
    }
};

// Float rules 1-5 (arc_verify.h), in fp64.  Returns true on mismatch; folds d
// into acc.ma and r into acc.rm (running maxima, NaN-ignoring via fmax).
__device__ __forceinline__ bool eval_f64(double x, double y, double at, double rt, ThreadAcc &acc) {
    const double d = fabs(x - y);             // NaN iff an operand is NaN (or Inf - Inf)
    const double ay = fabs(y);
    const double t = __dadd_rn(at, __dmul_rn(rt, ay));
    const bool match = (x == y) | ((x != x) & (y != y)) | ((ay < CUDART_INF) & (d <= t));
    acc.ma = fmax(acc.ma, d);                 // rule 1: x == y -> d = 0 (or NaN for equal Inf: ignored)
    // r > rm is only possible if d >= RN(rm * |y|) (monotone rounding); the
    // negated compare also lets NaN products through (rm = 0, |y| = Inf).
    if ((d > 0.0) & !(d < acc.rm * ay)) {
        const double r = (ay == CUDART_INF) ? CUDART_INF : d / ay;  // rule 4 / rule 5
        acc.rm = fmax(acc.rm, r);
    }
    return !match;
}

// eval_f64 with the optional N2 checks (arc_verify_check_t; readings R10/R11):
// not compared when |ref| <= min_value; a mismatch with lo <= out <= hi is
// ignored.  Either way: match, and d, r stay out of the maxima.
__device__ __forceinline__ bool eval_f64_checked(double x, double y, const SegHot &g, ThreadAcc &acc) {
    if (g.cflags == 0) return eval_f64(x, y, g.abs_tol, g.rel_tol, acc);
    if ((g.cflags & ARC_CHECK_MIN_VALUE) && fabs(y) <= g.minv) return false;
    if (g.cflags & ARC_CHECK_VALUE_BOUNDS) {
        const double d = fabs(x - y);
        const double t = __dadd_rn(g.abs_tol, __dmul_rn(g.rel_tol, fabs(y)));
        const bool match = (x == y) | ((x != x) & (y != y)) | ((fabs(y) < CUDART_INF) & (d <= t));
        if (!match && g.lo <= x && x <= g.hi) return false;
    }
    return eval_f64(x, y, g.abs_tol, g.rel_tol, acc);
}

// Exact pre-filter.  An element is finished without the
// fp64 rule iff
//     x == y    or    (d_f < RD(k * |y|)  and  d_f <= ma_f)
// where, in the element's own precision f (fp32 or fp64),
//     d_f = RN_f(|x - y|)  (one correctly rounded op on the exact difference;
//           for fp64 inputs this IS the oracle's d),
//     k   = min(rel_tol_f, rm_f, 1/4)  with rel_tol_f <= rel_tol and
//           rm_f <= rm (fp32: RD32(rel_tol) one ulp lower, RD32(rm (1 - 2^-40))),
//     ma_f = RD_f(ma).
// It then PROVES the fp64 rule's outcome:
//   match   : RD(k|y|) <= RN(rel_tol|y|) <= t, and (fp32) a float <= t is
//             <= RN32(t); RN is monotone, so |x - y| < t and d <= t;
//   no new max_rel: RN(d/|y|) > rm needs |x - y| > rm|y| (1 - 2^-52) > k|y|
//             >= RD(k|y|), and RN_f is monotone, so d_f >= RD(k|y|): excluded;
//   no new max_abs: d_f < |y|/4 makes x - y exact (Sterbenz), so d = d_f <= ma.
// Bounds only grow, so bounds read at the start of a tile are conservative.
template <typename T>
struct FastBounds {
    T k;      // min(rel_f, rm_f, 1/4)               (rel form)
    T kr;     // min(rm_f, 1/4)                      (abs form)
    T at;     // abs_f <= abs_tol                    (abs form)
    T ma;     // RD_f(ma)
};

__device__ __forceinline__ void refresh_bounds(const ThreadAcc &acc, float at_rd, float rt_rd,
                                               FastBounds<float> &b) {
    b.ma = __double2float_rd(acc.ma);
    b.kr = fminf(__double2float_rd(__dmul_rd(acc.rm, 1.0 - 0x1p-40)), 0.25f);
    b.k = fminf(rt_rd, b.kr);
    b.at = at_rd;
}
__device__ __forceinline__ void refresh_bounds(const ThreadAcc &acc, double at, double rt, FastBounds<double> &b) {
    b.ma = acc.ma;
    b.kr = fmin(acc.rm, 0.25);
    b.k = fmin(rt, b.kr);
    b.at = at;
}

// rel form (rel_tol > 0):  x == y  or  (d < RD(k|y|) and d <= ma_f)
// abs form (rel_tol = 0):  x == y  or  (d < abs_f and d < RD(kr|y|) and d <= ma_f)
// (kr <= 1/4 gives the Sterbenz exactness in both; abs_f <= abs_tol <= t.)
template <bool kRel>
__device__ __forceinline__ bool fast_ok(float x, float y, const FastBounds<float> &b) {
    const float d = fabsf(__fsub_rn(x, y));
    if constexpr (kRel) return (x == y) | ((d < __fmul_rd(b.k, fabsf(y))) & (d <= b.ma));
    else return (x == y) | ((d < b.at) & (d < __fmul_rd(b.kr, fabsf(y))) & (d <= b.ma));
}
template <bool kRel>
__device__ __forceinline__ bool fast_ok(double x, double y, const FastBounds<double> &b) {
    const double d = fabs(__dsub_rn(x, y));
    if constexpr (kRel) return (x == y) | ((d < __dmul_rd(b.k, fabs(y))) & (d <= b.ma));
    else return (x == y) | ((d < b.at) & (d < __dmul_rd(b.kr, fabs(y))) & (d <= b.ma));
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

// Running maxima are order-independent, so a thread may adopt any value that
// some thread of the same region has folded into its own maxima: the warp's
// maxima are valid filter bounds for every lane (the fold is idempotent).
// Called warp-uniformly.
__device__ __forceinline__ void share_bounds(ThreadAcc &acc) {
    acc.ma = warp_max_f64(acc.ma);
    acc.rm = warp_max_f64(acc.rm);
}

// Seed the running maxima once per region per thread: evaluate exactly the
// thread's element with the largest |x - y| and the one with the largest
// (approximate) |x - y| / |y| in its first tile, so that the fast pass starts
// with near-final bounds instead of flagging every record-breaking element.
// Evaluating an element here and again in the main pass is harmless: maxima
// are idempotent and the mismatch decision is taken by the main pass.
template <typename T, bool kAligned>
__device__ __forceinline__ void seed_bounds(const uint8_t *so, const uint8_t *sr, uint32_t off_o, uint32_t off_r,
                                            uint32_t cnt, int ctid, const SegHot &g, ThreadAcc &acc) {
    constexpr int EPV = 16 / sizeof(T);
    acc.seeded = true;
    float best_d = -1.f, best_r = -1.f;
    int bd = -1, br = -1;
    // The scan only picks which two elements to evaluate exactly, so it may be
    // approximate: fp32 arithmetic for fp32 data (no fp64 conversions), 16-byte
    // vector loads when the tile is aligned (f32x12 113.2 -> 110.9 us,
    // profiles/r02x_ab_seed_scan_fp32.log).  fp64 data keeps the plain scalar
    // scan (no gain there; its variants stay unchanged).
    if constexpr (!std::is_same<T, float>::value) {
        ARCV_UNROLL(ARCV_SEED_UNROLL)
        for (int b = 0; b < kVecPerThread * EPV; ++b) {
            const uint32_t e = (uint32_t)(((b / EPV) * kConsumerThreads + ctid) * EPV + (b % EPV));
            if (e >= cnt) continue;
            const T x = *reinterpret_cast<const T *>(so + off_o + e * sizeof(T));
            const T y = *reinterpret_cast<const T *>(sr + off_r + e * sizeof(T));
            const float d = (float)fabs((double)x - (double)y);
            const float r = __fdividef(d, fabsf((float)y) + 1e-37f);
            if (d > best_d && d < CUDART_INF_F) { best_d = d; bd = b; }
            if (r > best_r && r < CUDART_INF_F) { best_r = r; br = b; }
        }
    } else {
    ARCV_UNROLL(ARCV_EVAL_UNROLL)
    for (int k = 0; k < kVecPerThread; ++k) {
        const uint32_t v = k * kConsumerThreads + ctid;
        T xo[EPV], xr[EPV];
        if constexpr (kAligned) {
            const uint4 a = reinterpret_cast<const uint4 *>(so)[v];
            const uint4 c = reinterpret_cast<const uint4 *>(sr)[v];
            memcpy(xo, &a, 16);
            memcpy(xr, &c, 16);
        } else {
#pragma unroll
            for (int j = 0; j < EPV; ++j) {
                xo[j] = *reinterpret_cast<const T *>(so + off_o + (v * EPV + j) * sizeof(T));
                xr[j] = *reinterpret_cast<const T *>(sr + off_r + (v * EPV + j) * sizeof(T));
            }
        }
#pragma unroll
        for (int j = 0; j < EPV; ++j) {
            if (v * EPV + j >= cnt) continue;
            float d, r;
            if constexpr (std::is_same<T, float>::value) {
                d = fabsf(__fsub_rn(xo[j], xr[j]));
                r = __fdividef(d, fabsf(xr[j]) + 1e-37f);
            } else {
                d = (float)fabs(xo[j] - xr[j]);
                r = __fdividef(d, fabsf((float)xr[j]) + 1e-37f);
            }
            const int b = k * EPV + j;
            if (d > best_d && d < CUDART_INF_F) { best_d = d; bd = b; }
            if (r > best_r && r < CUDART_INF_F) { best_r = r; br = b; }
        }
    }
    }
    for (int q = 0; q < 2; ++q) {
        const int b = q == 0 ? bd : br;
        if (b < 0 || (q == 1 && br == bd)) continue;
        const uint32_t e = (uint32_t)(((b / EPV) * kConsumerThreads + ctid) * EPV + (b % EPV));
        const T x = *reinterpret_cast<const T *>(so + off_o + e * sizeof(T));
        const T y = *reinterpret_cast<const T *>(sr + off_r + e * sizeof(T));
        (void)eval_f64_checked((double)x, (double)y, g, acc);
    }
}

// Evaluate this thread's share of one tile; returns its number of mismatches
// (K1 needs only counts; the report phase re-derives the positions of the tiles it reports).
// Thread element order: bit k*EPV + j <-> tile element (k*256 + ctid)*EPV + j.
// Floats: a fast pass over all elements with the exact pre-filter, then the
// fp64 rule only for the (rare) flagged elements, re-read from the still-held
// shared-memory stage.
template <typename T, bool kFull, bool kAligned>
__device__ __forceinline__ uint32_t eval_tile(const uint8_t *so, const uint8_t *sr, uint32_t off_o, uint32_t off_r,
                                              uint32_t cnt, int ctid, const SegHot &g, ThreadAcc &acc) {
    constexpr int EPV = 16 / sizeof(T);
    constexpr bool kFloat = std::is_floating_point<T>::value;
    uint64_t slow = 0;
    uint32_t nmis = 0;
    uint32_t bmax = 0;  // u8 only: byte-wise running max |a - b|
    uint32_t dmax32 = 0;  // i32 only: running max |a - b| of this tile
    using RT = typename std::conditional<std::is_same<T, float>::value, float, double>::type;
    FastBounds<RT> fb;
    bool rel_form = true;
    if constexpr (kFloat) {
        if (!acc.seeded) {
            seed_bounds<T, kAligned>(so, sr, off_o, off_r, cnt, ctid, g, acc);
            share_bounds(acc);
#if !defined(ARCV_BLOCK_SEED) || ARCV_BLOCK_SEED
            // block-wide: every consumer warp seeds on this same tile (all
            // threads reset together at a region change), so the 8 warps'
            // seeded maxima -- folded values, valid bounds -- are pooled:
            // 8x the samples before the fast filter starts
            if ((ctid & 31) == 0) {
                g.seed_sh[ctid >> 5][0] = acc.ma;
                g.seed_sh[ctid >> 5][1] = acc.rm;
            }
            consumer_bar();
#pragma unroll
            for (int w = 0; w < kConsumerWarps; ++w) {
                acc.ma = fmax(acc.ma, g.seed_sh[w][0]);
                acc.rm = fmax(acc.rm, g.seed_sh[w][1]);
            }
            consumer_bar();  // the scratch is reused (flush_acc)
#endif
        }
        if constexpr (std::is_same<T, float>::value) {
            refresh_bounds(acc, g.at_rd, g.rt_rd, fb);
            rel_form = g.rt_rd > 0.f;
        } else {
            refresh_bounds(acc, g.abs_tol, g.rel_tol, fb);
            rel_form = g.rel_tol > 0.0;
        }
    }
    ARCV_UNROLL(ARCV_EVAL_UNROLL)
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
        uint32_t valid = (1u << EPV) - 1u;
        if constexpr (!kFull) {
            const uint32_t e0 = v * EPV;
            valid = e0 >= cnt ? 0u : (cnt - e0 >= (uint32_t)EPV ? valid : ((1u << (cnt - e0)) - 1u));
        }
        if (!kFloat && g.cflags != 0) {  // integers with N2 checks: plain scalar rule
            uint32_t mis = 0;
#pragma unroll
            for (int j = 0; j < EPV; ++j) {
                if (!((valid >> j) & 1u)) continue;
                const double xv = (double)xo[j], yv = (double)xr[j];
                if ((g.cflags & ARC_CHECK_MIN_VALUE) && fabs(yv) <= g.minv) continue;
                const uint64_t m = int_absdiff<T>(xo[j], xr[j]);
                if (m != 0 && (g.cflags & ARC_CHECK_VALUE_BOUNDS) && g.lo <= xv && xv <= g.hi) continue;
                acc.imax = m > acc.imax ? m : acc.imax;
                mis += (uint32_t)(m != 0);
            }
            nmis += mis;
        } else if constexpr (std::is_same<T, uint8_t>::value) {
            // bytes: SIMD-within-a-register.  |a-b| per byte is one native
            // VABSDIFF4.U8; a byte mismatches iff its |a-b| is nonzero (bit 7 of
            // each byte of nz); the byte-wise max (emulated vmaxu4) only runs for
            // words that hold a mismatch.
            uint32_t wa[4], wb[4];
            memcpy(wa, xo, 16);
            memcpy(wb, xr, 16);
#pragma unroll
            for (int w = 0; w < 4; ++w) {
                if constexpr (!kFull) {  // invalid bytes compare equal: spread 4 valid bits to bytes
                    const uint32_t vb = (valid >> (4 * w)) & 0xfu;
                    const uint32_t bm = ((vb * 0x00204081u) & 0x01010101u) * 0xffu;
                    wb[w] = (wb[w] & bm) | (wa[w] & ~bm);
                }
                const uint32_t ad = __vabsdiffu4(wa[w], wb[w]);
                const uint32_t nz = (((ad & 0x7f7f7f7fu) + 0x7f7f7f7fu) | ad) & 0x80808080u;
                nmis += __popc(nz);
                if (ad != 0u) bmax = __vmaxu4(bmax, ad);
            }
        } else if constexpr (kFloat) {
            uint32_t sl = 0;
            if (rel_form) {
#pragma unroll
                for (int j = 0; j < EPV; ++j) sl |= (uint32_t)(!fast_ok<true>((RT)xo[j], (RT)xr[j], fb)) << j;
            } else {
#pragma unroll
                for (int j = 0; j < EPV; ++j) sl |= (uint32_t)(!fast_ok<false>((RT)xo[j], (RT)xr[j], fb)) << j;
            }
            slow |= (uint64_t)(sl & valid) << (k * EPV);
        } else if constexpr (sizeof(T) == 4) {
            // int32: |a - b| <= 2^32 - 1 is exact in 32-bit unsigned arithmetic
            // (sad.s32 wraps mod 2^32); a per-tile 32-bit running max, folded
            // into the 64-bit accumulator once per tile.
            uint32_t mis = 0;
#pragma unroll
            for (int j = 0; j < EPV; ++j) {
                const uint32_t m = ((valid >> j) & 1u) ? __sad((int)xo[j], (int)xr[j], 0u) : 0u;
                dmax32 = max(dmax32, m);
                mis += min(m, 1u);
            }
            nmis += mis;
        } else {
            uint32_t mis = 0;
#pragma unroll
            for (int j = 0; j < EPV; ++j) {
                const uint64_t m = ((valid >> j) & 1u) ? int_absdiff<T>(xo[j], xr[j]) : 0ull;
                acc.imax = m > acc.imax ? m : acc.imax;
                mis += (uint32_t)(m != 0);
            }
            nmis += mis;
        }
    }
    if constexpr (!kFloat && sizeof(T) == 4) acc.imax = (uint64_t)dmax32 > acc.imax ? (uint64_t)dmax32 : acc.imax;
    if constexpr (std::is_same<T, uint8_t>::value) {
        const uint32_t m2 = __vmaxu4(bmax, bmax >> 16);
        const uint64_t mb = (uint64_t)max(m2 & 0xffu, (m2 >> 8) & 0xffu);
        acc.imax = mb > acc.imax ? mb : acc.imax;
    }
    if constexpr (kFloat) {
        if (slow) {  // rare: mismatches, specials, new maxima
            uint64_t m = slow;
            while (m) {
                const int b = __ffsll((long long)m) - 1;
                m &= m - 1;
                const uint32_t e = (uint32_t)(((b / EPV) * kConsumerThreads + ctid) * EPV + (b % EPV));
                const T x = *reinterpret_cast<const T *>(so + off_o + e * sizeof(T));
                const T y = *reinterpret_cast<const T *>(sr + off_r + e * sizeof(T));
                // the bounds grew since the fast pass: a re-check clears most of a
                // warm-up tile's flags without the fp64 rule
                if (rel_form ? fast_ok<true>((RT)x, (RT)y, fb) : fast_ok<false>((RT)x, (RT)y, fb)) continue;
                nmis += (uint32_t)eval_f64_checked((double)x, (double)y, g, acc);
                if constexpr (std::is_same<T, float>::value) refresh_bounds(acc, g.at_rd, g.rt_rd, fb);
                else refresh_bounds(acc, g.abs_tol, g.rel_tol, fb);
            }
        }
        // a lane's new maxima become the whole warp's filter bounds (the warp
        // then meets ~ln(32 n) record-breaking elements instead of ~ln(n) per lane)
        if (__any_sync(0xffffffffu, slow != 0)) share_bounds(acc);
    }
    return nmis;
}

template <typename T>
__device__ __forceinline__ uint32_t eval_tile_dispatch(const uint8_t *so, const uint8_t *sr, const StageInfo &si,
                                                       int ctid, const SegHot &g, ThreadAcc &acc) {
    constexpr uint32_t TE = kTileBytes / sizeof(T);
    const bool full = si.count == TE;
    const bool aligned = (si.off_o | si.off_r) == 0;
    if (full) {
        if (aligned) return eval_tile<T, true, true>(so, sr, 0, 0, TE, ctid, g, acc);
        return eval_tile<T, true, false>(so, sr, si.off_o, si.off_r, TE, ctid, g, acc);
    }
    if (aligned) return eval_tile<T, false, true>(so, sr, 0, 0, si.count, ctid, g, acc);
    return eval_tile<T, false, false>(so, sr, si.off_o, si.off_r, si.count, ctid, g, acc);
}

// A K1 specialised for a set of dtypes (bit 1 << ARC_* per dtype) compiles
// only those dtypes' tile evaluation: one dtype for single-region calls, the
// set a batch holds (kDtmFloatI32) for batches; kAllDtypes = any region.
template <int DTM = kAllDtypes>
__device__ __forceinline__ uint32_t eval_any(const uint8_t *so, const uint8_t *sr, const StageInfo &si, int ctid,
                                             const SegHot &g, ThreadAcc &acc) {
    if constexpr (DTM == (1 << ARC_F32)) return eval_tile_dispatch<float>(so, sr, si, ctid, g, acc);
    else if constexpr (DTM == (1 << ARC_F64)) return eval_tile_dispatch<double>(so, sr, si, ctid, g, acc);
    else if constexpr (DTM == (1 << ARC_I32)) return eval_tile_dispatch<int32_t>(so, sr, si, ctid, g, acc);
    else if constexpr (DTM == (1 << ARC_I64)) return eval_tile_dispatch<int64_t>(so, sr, si, ctid, g, acc);
    else if constexpr (DTM == (1 << ARC_U8)) return eval_tile_dispatch<uint8_t>(so, sr, si, ctid, g, acc);
    else {
        switch (g.dtype) {
            case ARC_F32:
                if constexpr ((DTM >> ARC_F32) & 1) return eval_tile_dispatch<float>(so, sr, si, ctid, g, acc);
                else return 0u;  // not launched with this kernel
            case ARC_F64:
                if constexpr ((DTM >> ARC_F64) & 1) return eval_tile_dispatch<double>(so, sr, si, ctid, g, acc);
                else return 0u;
            case ARC_I32:
                if constexpr ((DTM >> ARC_I32) & 1) return eval_tile_dispatch<int32_t>(so, sr, si, ctid, g, acc);
                else return 0u;
            case ARC_I64:
                if constexpr ((DTM >> ARC_I64) & 1) return eval_tile_dispatch<int64_t>(so, sr, si, ctid, g, acc);
                else return 0u;
            default:
                if constexpr ((DTM >> ARC_U8) & 1) return eval_tile_dispatch<uint8_t>(so, sr, si, ctid, g, acc);
                else return 0u;
        }
    }
}

// ------------------------------------------------------------ tile loading
// Plan the bulk copies of segment-local tile `lt`: 16-byte-aligned windows that
// cover the tile in each array (arbitrary element alignment; the extra bytes
// lie in the same 16-byte granules as valid ones, hence in mapped pages).
__device__ __forceinline__ void plan_tile(const Seg &g, uint64_t lt, StageInfo &si, uintptr_t &ao, uint32_t &nbo,
                                          uintptr_t &ar, uint32_t &nbr) {
    const uint32_t es = elem_size(g.dtype);
    const uint64_t te = kTileBytes / es;
    const uint64_t e0 = lt * te;
    const uint64_t rem = g.n - e0;
    const uint32_t cnt = (uint32_t)(rem < te ? rem : te);
    const uintptr_t bo = reinterpret_cast<uintptr_t>(g.out) + e0 * es;
    const uintptr_t br = reinterpret_cast<uintptr_t>(g.ref) + e0 * es;
    ao = bo & ~(uintptr_t)15;
    ar = br & ~(uintptr_t)15;
    nbo = (uint32_t)(((bo + (uint64_t)cnt * es + 15) & ~(uintptr_t)15) - ao);
    nbr = (uint32_t)(((br + (uint64_t)cnt * es + 15) & ~(uintptr_t)15) - ar);
    si.elem_begin = e0;
    si.count = cnt;
    si.off_o = (uint32_t)(bo - ao);
    si.off_r = (uint32_t)(br - ar);
}

__device__ __forceinline__ uint64_t evict_first_policy() {
    uint64_t policy;
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(policy));
    return policy;
}

__device__ __forceinline__ uint32_t find_seg(const Seg *segs, uint32_t n, uint64_t t) {
    uint32_t lo = 0, hi = n;  // last seg with tile_begin <= t
    while (hi - lo > 1) {
        const uint32_t mid = (lo + hi) >> 1;
        if (segs[mid].tile_begin <= t) lo = mid; else hi = mid;
    }
    return lo;
}

// ------------------------------------------------------------ accumulators
// Block-wide (consumer threads) reduction of the thread accumulators into the
// region's global accumulator slot.
__device__ __forceinline__ void flush_acc(Acc *acc_base, uint32_t slot, uint32_t dtype, ThreadAcc &acc, int ctid,
                                          uint64_t (*s_u)[2], double (*s_d)[2]) {
    const int lane = ctid & 31, cw = ctid >> 5;
    const bool is_float = dtype == ARC_F32 || dtype == ARC_F64;
    const double mabs = is_float ? acc.ma : __ull2double_rn(acc.imax);
    const uint64_t c = warp_sum_u64(acc.count);
    const double wa = warp_max_f64(mabs);
    const double wr = warp_max_f64(acc.rm);
    if (lane == 0) {
        s_u[cw][0] = c;
        s_d[cw][0] = wa;
        s_d[cw][1] = wr;
    }
    consumer_bar();
    if (ctid == 0) {
        uint64_t tc = 0;
        double ta = 0.0, tr = 0.0;
        for (int w = 0; w < kConsumerWarps; ++w) {
            tc += s_u[w][0];
            ta = fmax(ta, s_d[w][0]);
            tr = fmax(tr, s_d[w][1]);
        }
        Acc *a = acc_base + slot;
        if (tc) atomicAdd(&a->count, (unsigned long long)tc);
        if (ta > 0.0) atomicMax(&a->max_abs_bits, (unsigned long long)__double_as_longlong(ta));
        if (tr > 0.0) atomicMax(&a->max_rel_bits, (unsigned long long)__double_as_longlong(tr));
    }
    consumer_bar();
    acc.reset();
}

// The last CTA of the launch copies the accumulators to the result slots and
// clears them for the next call (monotonic done counter, host-tracked base).
// It then stores the call's sequence number to a mapped host word, which the
// host polls instead of a stream synchronise; system-scope fences order report
// entries written to pinned host memory (report phase, `wrote_host`) and the results
// before that word.
__device__ __forceinline__ bool last_cta(const Params &p, int tid, int nthreads, int *s_last, bool wrote_host,
                                         unsigned long long base) {
    if (tid == 0) {
        if (wrote_host) fence_sys();
        else fence_gpu();
        const unsigned long long prev = atomicAdd(p.done, 1ull);
        *s_last = (prev - base) == (unsigned long long)(gridDim.x - 1);
    }
    if (nthreads == kConsumerThreads) consumer_bar(); else __syncthreads();
    return *s_last != 0;
}

// `fenced` = false for launches that wrote no report entry to host memory (a
// clean or count-only call): the slots validate themselves (slot_tag), so the
// completion word needs no system fence -- one PCIe round trip (~3 us) less
// in the last CTA.  With entries written over PCIe the cumulative system fence
// orders them (and the slots) before the word.
// `n_nz`: the launch's final pool length when the caller has it (saves a
// dependent load on the completion path), else ~0u.
// `pre` (optional): slot `tid`'s accumulators, already read by the caller after
// every CTA had flushed (the report phase loads them while its tiles land), so
// the publishing CTA does not wait for them.
__device__ __forceinline__ void publish(const Params &p, int tid, int nthreads, bool fenced = true,
                                        uint32_t n_nz = ~0u, const Acc *pre = nullptr) {
    {
        fence_gpu();
        // the report phase's path (the host re-applies direct_route with it)
        if (n_nz == ~0u) n_nz = *(volatile uint32_t *)p.nz_cnt;
        const unsigned long long route = (p.k2 && n_nz <= (uint32_t)kPoolCap) ? kRoutePool : 0ull;
        for (uint32_t k = tid; k < p.n_acc; k += nthreads) {
            Acc a;
            if (pre != nullptr && k == (uint32_t)tid) {
                a = *pre;
            } else {
                a.count = __ldcg(&p.acc[k].count);
                a.max_abs_bits = __ldcg(&p.acc[k].max_abs_bits);
                a.max_rel_bits = __ldcg(&p.acc[k].max_rel_bits);
            }
            a.pad = slot_tag(p.seq, route, a.count, a.max_abs_bits, a.max_rel_bits);
            p.result[k] = a;
            if (p.mirror) p.mirror[k] = a;
            p.acc[k].count = 0;
            p.acc[k].max_abs_bits = 0;
            p.acc[k].max_rel_bits = 0;
        }
        if (p.done_flag) {
            if (nthreads == kConsumerThreads) consumer_bar(); else __syncthreads();
            if (tid == 0) {
                if (fenced) fence_sys();
                *(volatile unsigned long long *)p.done_flag = p.seq;
            }
        }
    }
}

__device__ __forceinline__ void finalize_launch(const Params &p, int tid, int nthreads, int *s_last,
                                                bool wrote_host, unsigned long long base, bool do_publish = true) {
    if (last_cta(p, tid, nthreads, s_last, wrote_host, base) && do_publish) publish(p, tid, nthreads);
}

// Sharded call with the exchange fused into K1 (p.xfused; K1 is a cooperative
// launch): the CTA that published the local result (`leader`) publishes the
// rank's header and flags, then every CTA runs the exchange body -- wait for
// the peers' flags, merge its share of the global report, and the last one
// writes the global result and the completion word.  Scratch: the (free)
// stage memory.
__device__ __forceinline__ void exchange_tail(const Params &p, int tid, bool leader, uint8_t *smem) {
    if (leader && tid == 0) {
        // written by publish() in this CTA or (clean fused call) in the CTA that
        // arrived last at the grid barrier, released before its done count
        fence_gpu();  // acquire side of that release (the done count was observed above)
        const Acc *m = p.mirror;
        peer_publish_header(p.x, __ldcg(&m->count), __ldcg(&m->max_abs_bits), __ldcg(&m->max_rel_bits));
    }
    peer_exchange_body(p.x, tid, *reinterpret_cast<ExShared *>(smem));
}

// ------------------------------------------------------ report-phase helpers
// Exclusive scan over the 256 consumer threads (named barrier 1; `tid` = the
// consumer index, so K1's consumer warps can run it too) of a u64; returns the
// exclusive prefix, writes the block total to *total.
__device__ __forceinline__ uint64_t block_excl_scan(uint64_t v, uint64_t *s_w, uint64_t *total, int tid) {
    const int lane = tid & 31, w = tid >> 5;
    uint64_t inc = v;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const uint64_t y = __shfl_up_sync(0xffffffffu, inc, o);
        if (lane >= o) inc += y;
    }
    if (lane == 31) s_w[w] = inc;
    consumer_bar();
    uint64_t base = 0, tot = 0;
#pragma unroll
    for (int k = 0; k < kConsumerWarps; ++k) {
        const uint64_t x = s_w[k];
        base += (k < w) ? x : 0ull;
        tot += x;
    }
    consumer_bar();
    *total = tot;
    return base + inc - v;
}

// Writes this tile's mismatches with global report rank excl + in-tile rank,
// for ranks < max_report.  In-tile order = element index order = (k, tid, j).
// `obuf` non-null (a dense tile going to pinned host memory): only the tile's
// in-tile ranks [rlo, rhi) are written, in rounds of kOutEntries entries staged
// in shared memory and stored as consecutive 8-byte words (one warp store =
// 256 contiguous bytes, i.e. full PCIe write packets instead of 24-byte
// scatter).  Called by all 256 consumer threads (it synchronises them).
constexpr int kOutEntries = 1024;
template <typename T>
__device__ __noinline__ void compact_tile(const Seg &g, uint64_t si_elem_begin, uint32_t si_off_o, uint32_t si_off_r, const uint8_t *so, const uint8_t *sr,
                                          uint64_t mask, uint64_t excl, uint64_t *s_w, int tid, uint64_t rlo,
                                          uint64_t rhi, arc_mismatch_t *obuf) {
    constexpr int EPV = 16 / sizeof(T);
    constexpr uint64_t kGroup = EPV == 64 ? ~0ull : ((1ull << EPV) - 1ull);
    uint64_t packed = 0;  // 4 x 16-bit per-k counts; field totals <= 4096 (no carries)
#pragma unroll
    for (int k = 0; k < kVecPerThread; ++k)
        packed |= (uint64_t)__popcll(mask & (kGroup << (k * EPV))) << (16 * k);
    uint64_t total;
    const uint64_t ex = block_excl_scan(packed, s_w, &total, tid);
    arc_mismatch_t *const rep = (excl & kDirectBit) ? g.report_alias : g.report;
    excl &= ~kDirectBit;
    if (obuf) {
        const uint64_t lim = g.max_report > excl ? g.max_report - excl : 0ull;  // reported ranks < lim
        const uint64_t hi = rhi < lim ? rhi : lim;
        for (uint64_t r0 = rlo; r0 < hi; r0 += kOutEntries) {  // uniform
            const uint64_t r1 = r0 + kOutEntries < hi ? r0 + kOutEntries : hi;
            uint64_t m = mask;
            while (m) {
                const int b = __ffsll((long long)m) - 1;
                m &= m - 1;
                const int k = b / EPV, j = b % EPV;
                uint64_t rank = ((ex >> (16 * k)) & 0xffffull) +
                                (uint64_t)__popcll(mask & (((1ull << j) - 1ull) << (k * EPV)));
                for (int kk = 0; kk < k; ++kk) rank += (total >> (16 * kk)) & 0xffffull;
                if (rank >= r0 && rank < r1) {
                    const uint32_t te = (uint32_t)((k * kConsumerThreads + tid) * EPV + j);
                    arc_mismatch_t e;
                    e.index = g.index_base + si_elem_begin + te;
                    e.out_bits = raw_bits<T>(*reinterpret_cast<const T *>(so + si_off_o + te * sizeof(T)));
                    e.ref_bits = raw_bits<T>(*reinterpret_cast<const T *>(sr + si_off_r + te * sizeof(T)));
                    obuf[rank - r0] = e;
                }
            }
            consumer_bar();
            const uint64_t nw = 3 * (r1 - r0);
            const unsigned long long *src = reinterpret_cast<const unsigned long long *>(obuf);
            unsigned long long *dst = reinterpret_cast<unsigned long long *>(rep + excl + r0);
            for (uint64_t w = tid; w < nw; w += kConsumerThreads) dst[w] = src[w];
            consumer_bar();  // obuf is reused
        }
        return;
    }
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
            const uint32_t te = (uint32_t)((k * kConsumerThreads + tid) * EPV + j);  // tile element
            const T xo = *reinterpret_cast<const T *>(so + si_off_o + te * sizeof(T));  // from the stage
            const T xr = *reinterpret_cast<const T *>(sr + si_off_r + te * sizeof(T));
            arc_mismatch_t *dst = rep + gi;
            dst->index = g.index_base + si_elem_begin + te;
            dst->out_bits = raw_bits<T>(xo);
            dst->ref_bits = raw_bits<T>(xr);
        }
    }
}

// ----------------------------------------------------- report phase: mask only
// The report phase needs only the mismatch decision of each element of a re-read tile (the
// maxima were taken by K1).  A compact, non-unrolled loop of the plain rule:
// small code matters here because every CTA executes it cold, once.
// The decision is the same rule K1 applies (its fast path only ever proves
// matches), so the in-tile ranks agree with K1's counts.
// Scalars by value: references to SegHot / StageInfo would put them in local
// memory (the function is not inlined) and reload them every iteration.
// -DARCV_MASK_UNROLL=N: unroll the mask loops N-fold (A/B builds; default 1:
// compact code, cold once per CTA).
#ifndef ARCV_MASK_UNROLL
#define ARCV_MASK_UNROLL 1
#endif
template <typename T>
__device__ __noinline__ uint64_t mask_tile(const uint8_t *so, const uint8_t *sr, uint32_t count, uint32_t off_o,
                                           uint32_t off_r, int tid, double abs_tol, double rel_tol, uint32_t cflags,
                                           double minv, double lo, double hi) {
    constexpr int EPV = 16 / sizeof(T);
    uint64_t mask = 0;
    if constexpr (!std::is_floating_point<T>::value) {
        if (cflags == 0) {  // integers: plain equality
#pragma unroll 4
            for (int b = 0; b < kVecPerThread * EPV; ++b) {
                const uint32_t e = (uint32_t)(((b / EPV) * kConsumerThreads + tid) * EPV + (b % EPV));
                if (e >= count) continue;
                const T xo = *reinterpret_cast<const T *>(so + off_o + e * sizeof(T));
                const T yr = *reinterpret_cast<const T *>(sr + off_r + e * sizeof(T));
                mask |= (uint64_t)(xo != yr) << b;
            }
            return mask;
        }
    }
    ARCV_UNROLL(ARCV_MASK_UNROLL)
    for (int b = 0; b < kVecPerThread * EPV; ++b) {
        const uint32_t e = (uint32_t)(((b / EPV) * kConsumerThreads + tid) * EPV + (b % EPV));
        if (e >= count) continue;
        const T xo = *reinterpret_cast<const T *>(so + off_o + e * sizeof(T));
        const T yr = *reinterpret_cast<const T *>(sr + off_r + e * sizeof(T));
        const double x = (double)xo, y = (double)yr;
        if ((cflags & ARC_CHECK_MIN_VALUE) && fabs(y) <= minv) continue;
        bool mis;
        if constexpr (std::is_floating_point<T>::value) {
            const double d = fabs(x - y);
            const double t = __dadd_rn(abs_tol, __dmul_rn(rel_tol, fabs(y)));
            mis = !((x == y) | ((x != x) & (y != y)) | ((fabs(y) < CUDART_INF) & (d <= t)));
        } else {
            mis = xo != yr;
        }
        if (mis && (cflags & ARC_CHECK_VALUE_BOUNDS) && lo <= x && x <= hi) mis = false;
        mask |= (uint64_t)mis << b;
    }
    return mask;
}

template <typename G>
__device__ __forceinline__ uint64_t mask_any(const uint8_t *so, const uint8_t *sr, const StageInfo &si, int tid,
                                             const G &g) {
#define ARCV_MASK(T) mask_tile<T>(so, sr, si.count, si.off_o, si.off_r, tid, g.abs_tol, g.rel_tol, g.cflags, \
                                  g.minv, g.lo, g.hi)
    switch (g.dtype) {
        case ARC_F32: return ARCV_MASK(float);
        case ARC_F64: return ARCV_MASK(double);
        case ARC_I32: return ARCV_MASK(int32_t);
        case ARC_I64: return ARCV_MASK(int64_t);
        default: return ARCV_MASK(uint8_t);
    }
#undef ARCV_MASK
}

// ------------------------------------------------------- report phase: compact
__device__ __forceinline__ unsigned long long ld_acquire_u64(const unsigned long long *p) {
    unsigned long long v;
    asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}

// Software grid barrier (K1-with-report and K2 are cooperative launches, so all CTAs are
// co-resident).  Monotonic counter; the host tracks each launch's base.
// `tid` = consumer index; the 256 consumer threads synchronise on barrier 1.
__device__ __forceinline__ void grid_barrier(unsigned long long *ctr, unsigned long long base, int tid) {
    consumer_bar();
    if (tid == 0) {
        fence_gpu();
        atomicAdd(ctr, 1ull);
        while (ld_acquire_u64(ctr) - base < (unsigned long long)gridDim.x) __nanosleep(32);
    }
    consumer_bar();
}

// ---- half-block variants: warps 0-3 and 4-7 each handle one tile at once ----
// (a CTA owning two report tiles processes them concurrently; 128 threads per
// tile, 8 vectors per thread: element e = ((b / EPV) * 128 + gt) * EPV + b % EPV.
// Not for u8: 8 x 16 mismatch bits do not fit the 64-bit mask.)
__device__ __forceinline__ void half_bar(int grp) {
    asm volatile("bar.sync %0, 128;" ::"r"(2 + grp) : "memory");
}
// exclusive scan of two u64 over the 128 threads of half `grp`; totals out
__device__ __forceinline__ void half_excl_scan2(uint64_t v0, uint64_t v1, uint64_t *s_w, int gt, int grp,
                                                uint64_t *ex0, uint64_t *ex1, uint64_t *t0, uint64_t *t1) {
    const int lane = gt & 31, w = gt >> 5;
    uint64_t a = v0, c = v1;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const uint64_t ya = __shfl_up_sync(0xffffffffu, a, o);
        const uint64_t yc = __shfl_up_sync(0xffffffffu, c, o);
        if (lane >= o) {
            a += ya;
            c += yc;
        }
    }
    if (lane == 31) {
        s_w[2 * w] = a;
        s_w[2 * w + 1] = c;
    }
    half_bar(grp);
    uint64_t ba = 0, bc = 0, ta = 0, tc = 0;
#pragma unroll
    for (int k = 0; k < 4; ++k) {
        const uint64_t xa = s_w[2 * k], xc = s_w[2 * k + 1];
        ba += (k < w) ? xa : 0ull;
        bc += (k < w) ? xc : 0ull;
        ta += xa;
        tc += xc;
    }
    half_bar(grp);
    *ex0 = ba + a - v0;
    *ex1 = bc + c - v1;
    *t0 = ta;
    *t1 = tc;
}

template <typename T>
__device__ __noinline__ uint64_t mask_tile_half(const uint8_t *so, const uint8_t *sr, uint32_t count, uint32_t off_o,
                                                uint32_t off_r, int gt, double abs_tol, double rel_tol,
                                                uint32_t cflags, double minv, double lo, double hi) {
    constexpr int EPV = 16 / sizeof(T);
    uint64_t mask = 0;
    ARCV_UNROLL(ARCV_MASK_UNROLL)
    for (int b = 0; b < 2 * kVecPerThread * EPV; ++b) {
        const uint32_t e = (uint32_t)(((b / EPV) * (kConsumerThreads / 2) + gt) * EPV + (b % EPV));
        if (e >= count) continue;
        const T xo = *reinterpret_cast<const T *>(so + off_o + e * sizeof(T));
        const T yr = *reinterpret_cast<const T *>(sr + off_r + e * sizeof(T));
        const double x = (double)xo, y = (double)yr;
        if ((cflags & ARC_CHECK_MIN_VALUE) && fabs(y) <= minv) continue;
        bool mis;
        if constexpr (std::is_floating_point<T>::value) {
            const double d = fabs(x - y);
            const double t = __dadd_rn(abs_tol, __dmul_rn(rel_tol, fabs(y)));
            mis = !((x == y) | ((x != x) & (y != y)) | ((fabs(y) < CUDART_INF) & (d <= t)));
        } else {
            mis = xo != yr;
        }
        if (mis && (cflags & ARC_CHECK_VALUE_BOUNDS) && lo <= x && x <= hi) mis = false;
        mask |= (uint64_t)mis << b;
    }
    return mask;
}

template <typename T>
__device__ __noinline__ void compact_tile_half(const Seg &g, uint64_t si_elem_begin, uint32_t si_off_o, uint32_t si_off_r, const uint8_t *so,
                                               const uint8_t *sr, uint64_t mask, uint64_t excl, uint64_t *s_w,
                                               int gt, int grp) {
    constexpr int EPV = 16 / sizeof(T);
    constexpr int NV = 2 * kVecPerThread;  // 8 vectors: fields 0-3 in p0, 4-7 in p1
    constexpr uint64_t kGroup = (1ull << EPV) - 1ull;
    uint64_t p0 = 0, p1 = 0;  // 4 x 16-bit per-k counts each; totals <= 128 * 4
#pragma unroll
    for (int k = 0; k < NV; ++k) {
        const uint64_t c = (uint64_t)__popcll(mask & (kGroup << (k * EPV)));
        if (k < 4) p0 |= c << (16 * k);
        else p1 |= c << (16 * (k - 4));
    }
    uint64_t ex0, ex1, t0, t1;
    half_excl_scan2(p0, p1, s_w, gt, grp, &ex0, &ex1, &t0, &t1);
    arc_mismatch_t *const rep = (excl & kDirectBit) ? g.report_alias : g.report;
    excl &= ~kDirectBit;
    uint64_t m = mask;
    while (m) {
        const int bpos = __ffsll((long long)m) - 1;
        m &= m - 1;
        const int k = bpos / EPV, j = bpos % EPV;
        uint64_t rank = (uint64_t)__popcll(mask & (((1ull << j) - 1ull) << (k * EPV)));
        rank += k < 4 ? ((ex0 >> (16 * k)) & 0xffffull) : ((ex1 >> (16 * (k - 4))) & 0xffffull);
        for (int kk = 0; kk < k; ++kk)
            rank += kk < 4 ? ((t0 >> (16 * kk)) & 0xffffull) : ((t1 >> (16 * (kk - 4))) & 0xffffull);
        const uint64_t gi = excl + rank;
        if (gi < g.max_report) {
            const uint32_t te = (uint32_t)((k * (kConsumerThreads / 2) + gt) * EPV + j);
            const T xo = *reinterpret_cast<const T *>(so + si_off_o + te * sizeof(T));
            const T xr = *reinterpret_cast<const T *>(sr + si_off_r + te * sizeof(T));
            arc_mismatch_t *dst = rep + gi;
            dst->index = g.index_base + si_elem_begin + te;
            dst->out_bits = raw_bits<T>(xo);
            dst->ref_bits = raw_bits<T>(xr);
        }
    }
}

__device__ __forceinline__ void emit_half_any(const Seg &g, const StageInfo &si, const uint8_t *so, uint64_t excl,
                                              uint64_t *s_w, int gt, int grp) {
#define ARCV_HALF(T)                                                                                          \
    {                                                                                                         \
        const uint64_t mk = mask_tile_half<T>(so, so + kStageArrayBytes, si.count, si.off_o, si.off_r, gt,     \
                                              g.abs_tol, g.rel_tol, g.cflags, g.minv, g.lo, g.hi);            \
        compact_tile_half<T>(g, si.elem_begin, si.off_o, si.off_r, so, so + kStageArrayBytes, mk, excl, s_w, gt, grp);                      \
    }
    switch (g.dtype) {
        case ARC_F32: ARCV_HALF(float) break;
        case ARC_F64: ARCV_HALF(double) break;
        case ARC_I32: ARCV_HALF(int32_t) break;
        default: ARCV_HALF(int64_t) break;
    }
#undef ARCV_HALF
}

__device__ __forceinline__ void compact_any(const Seg &g, const StageInfo &si, const uint8_t *so, const uint8_t *sr,
                                            uint64_t mask, uint64_t excl, uint64_t *s_w, int tid, uint64_t rlo,
                                            uint64_t rhi, arc_mismatch_t *obuf) {
    switch (g.dtype) {
        case ARC_F32: compact_tile<float>(g, si.elem_begin, si.off_o, si.off_r, so, sr, mask, excl, s_w, tid, rlo, rhi, obuf); break;
        case ARC_F64: compact_tile<double>(g, si.elem_begin, si.off_o, si.off_r, so, sr, mask, excl, s_w, tid, rlo, rhi, obuf); break;
        case ARC_I32: compact_tile<int32_t>(g, si.elem_begin, si.off_o, si.off_r, so, sr, mask, excl, s_w, tid, rlo, rhi, obuf); break;
        case ARC_I64: compact_tile<int64_t>(g, si.elem_begin, si.off_o, si.off_r, so, sr, mask, excl, s_w, tid, rlo, rhi, obuf); break;
        default: compact_tile<uint8_t>(g, si.elem_begin, si.off_o, si.off_r, so, sr, mask, excl, s_w, tid, rlo, rhi, obuf); break;
    }
}

// The report phase (a5): which tiles' mismatches enter the report, re-read them,
// write their entries in ascending index order.  Runs either in K2 (its own
// cooperative launch after K1) or -- fused, the default -- in K1's consumer
// warps after a grid barrier, so the report costs no second launch.
//
// Two ways to find the report tiles:
// Pool path (the common, sparse case: K1 listed <= kPoolCap nonzero tiles):
//   pool entry k is handled by CTA k mod grid.  A CTA issues the bulk re-reads
//   of its first two entries at once, then gets their exclusive prefixes in ONE
//   pass over the pool (sum of the counts of listed tiles of the same segment
//   with a smaller index; read from L2) and one block reduction; no grid barrier.
// Group path (dense: the list overflowed):
//   Phase A: every CTA scans the group counters of each reporting segment (a few
//   KB); nonzero groups are owned round-robin by their ordinal, the owner scans
//   the group's 256 tile counts, appends every tile whose exclusive prefix is
//   below max_report to the active list {seg, tile, prefix}.  Grid barrier.
// Then each CTA re-reads its active tiles through a 2-stage bulk-copy ring,
// re-evaluates them, and writes their mismatches at report positions
// prefix + in-tile rank.  Tile counts are cleared for the next call by whoever
// handled the tile / group.
// `smem`: >= kReportSmem bytes of dynamic shared memory (2 stages + RepShared);
// `tid`: consumer index 0..255 (named barrier 1).  Counter contract: adds
// exactly gridDim.x to p.gbar, and (p.finalize) exactly gridDim.x to p.done
// above `done_base`; the last CTA publishes unless `k1_published`.
struct RepShared {
    uint64_t bar[2];
    uint64_t w[kConsumerWarps];
    uint64_t red[kConsumerWarps][4];
    uint64_t hw[2][8];  // half-block scans (two tiles at once)
    uint64_t owned_pre[kGroupTiles];
    uint32_t owned[kGroupTiles];
    uint32_t n;
    int last;
    int wrote;  // this CTA wrote report entries to pinned host memory
};
// [stage 0][stage 1][RepShared][out buffer: kOutEntries entries]
constexpr int kReportSmem = 2 * kStageBytes + (int)sizeof(RepShared) + kOutEntries * (int)sizeof(arc_mismatch_t);

template <bool XF>
__device__ __forceinline__ void report_phase(const Params &p, const Seg *segs, uint8_t *smem, int tid,
                                             unsigned long long done_base, bool k1_published_if_empty,
                                             uint32_t n_nz_known = ~0u) {
    RepShared &sh = *reinterpret_cast<RepShared *>(smem + 2 * kStageBytes);
    if (tid == 0) {
        ARCV_STAMP(1, 1);
        sh.wrote = 0;
        mbar_init(&sh.bar[0], 1);
        mbar_init(&sh.bar[1], 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    consumer_bar();
    const uint64_t policy = evict_first_policy();
    constexpr uint64_t kLtMask = (1ull << 40) - 1;
    uint32_t phase = 0u;  // bit st: the parity stage st's barrier waits for next (no local array)
    auto issue = [&](uint64_t key, int st) {
        const Seg &g = segs[key >> 40];
        StageInfo si;
        uintptr_t ao, ar;
        uint32_t nbo, nbr;
        plan_tile(g, key & kLtMask, si, ao, nbo, ar, nbr);
        uint8_t *dst = smem + (size_t)st * kStageBytes;
        mbar_arrive_expect_tx(&sh.bar[st], nbo + nbr);
        bulk_g2s(dst, reinterpret_cast<const void *>(ao), nbo, &sh.bar[st], policy);
        bulk_g2s(dst + kStageArrayBytes, reinterpret_cast<const void *>(ar), nbr, &sh.bar[st], policy);
    };
    // wait for tile `key` in stage st, write its entries from report rank excl.
    // A region with a report_alias (pinned host memory, the caller's or the
    // library's staging for a pageable buffer) gets its entries written there
    // directly over PCIe when direct_route() holds -- K1's final count and the
    // path taken decide it; the host applies the same rule to the published
    // slot.  `tc` = the tile's count (pool path; 0 if unknown): a dense tile
    // going straight to pinned memory is written through the shared-memory out
    // buffer as coalesced words.
    arc_mismatch_t *const obuf = reinterpret_cast<arc_mismatch_t *>(smem + 2 * kStageBytes + sizeof(RepShared));
    auto emit = [&](uint64_t key, uint64_t excl, int st, bool pool, uint64_t tc, bool stamp = false) {
        const Seg &g = segs[key >> 40];
        const bool direct = direct_route(g.report_alias != nullptr, g.flags, __ldcg(&p.acc[g.acc_slot].count),
                                         g.max_report, g.alias_cap, pool);
        StageInfo si;
        uintptr_t ao, ar;
        uint32_t nbo, nbr;
        plan_tile(g, key & kLtMask, si, ao, nbo, ar, nbr);
        mbar_wait(&sh.bar[st], (phase >> st) & 1u);
        phase ^= 1u << st;
        if (tid == 0 && stamp) ARCV_STAMP(1, 4);
        if (excl < g.max_report) {  // uniform
            if ((direct || (g.flags & kSegReportHost)) && tid == 0) sh.wrote = 1;
            const uint8_t *so = smem + (size_t)st * kStageBytes;
            const uint64_t mask = mask_any(so, so + kStageArrayBytes, si, tid, g);
            if (tid == 0 && stamp) ARCV_STAMP(1, 5);
            const bool staged = direct && tc > kStagedMin;
            compact_any(g, si, so, so + kStageArrayBytes, mask, excl | (direct ? kDirectBit : 0ull), sh.w, tid,
                        0ull, staged ? tc : ~0ull, staged ? obuf : nullptr);
        }
        consumer_bar();  // stage `st` and sh.w are reused
        if (tid == 0 && stamp) ARCV_STAMP(1, 2);
    };

    // the final pool length: the fused tail read it after the grid barrier already
    const uint32_t n_nz = n_nz_known != ~0u ? n_nz_known : *(volatile uint32_t *)p.nz_cnt;
    // this thread's result slot, final since every CTA flushed before the barrier:
    // read now, off the publishing CTA's critical path
    Acc pre_acc;
    const bool have_pre = p.finalize && (uint32_t)tid < p.n_acc;
    if (have_pre) {
        pre_acc.count = __ldcg(&p.acc[tid].count);
        pre_acc.max_abs_bits = __ldcg(&p.acc[tid].max_abs_bits);
        pre_acc.max_rel_bits = __ldcg(&p.acc[tid].max_rel_bits);
    }
    const uint32_t G = gridDim.x, b = blockIdx.x;
    if (n_nz <= (uint32_t)kPoolCap) {
        // ------------------------------------------------------ pool path
        // arrive on the grid-barrier counter without waiting (host base += grid)
        if (tid == 0) atomicAdd(p.gbar, 1ull);
        // (Round 2 measured splitting a dense tile across several CTAs: C2B
        // -10 us per call, but any form of that code in K1's tail -- inline or
        // out of line -- changed the stream loop's code generation and cost
        // sparse calls ~2 us and C3 ~5 us (profiles/r02ah_ab.log,
        // r02aj_ab.log); dense direct tiles are written by one CTA, staged.)
        const uint32_t n_items = n_nz;
#if defined(ARCV_TAIL_REPS)
      // diagnostic: run the (idempotent) pool path again, stamps from the last run
      for (int rep_ = 0; rep_ < ARCV_TAIL_REPS; ++rep_) {
        consumer_bar();
        if (tid == 0) ARCV_STAMP(1, 8);
#endif
        const uint32_t n_own = n_items > b ? (n_items - b + G - 1) / G : 0u;
        auto entry_of = [&](uint32_t j) { return b + j * G; };  // my j-th pool entry
        const ulonglong2 *nzl = reinterpret_cast<const ulonglong2 *>(p.nz_list);
        // One round trip for everything the prefixes and the first re-reads
        // need: the CTA's first two pool entries (every thread: they are also
        // the keys of the prefix pass) and the whole pool in registers (entry
        // tid + u * 256 = {seg << 40 | tile, count}; absent entries never
        // match), all loads in flight before thread 0 issues the re-reads.
        ulonglong2 kv[2] = {make_ulonglong2(~0ull - 1, 0ull), make_ulonglong2(~0ull - 1, 0ull)};
        if (n_own > 0) kv[0] = __ldcg(nzl + entry_of(0));
        if (n_own > 1) kv[1] = __ldcg(nzl + entry_of(1));
        constexpr int kPer = kPoolCap / kConsumerThreads;
        uint64_t pk[kPer], pc[kPer];
#pragma unroll
        for (int u = 0; u < kPer; ++u) {
            const uint32_t i = (uint32_t)tid + (uint32_t)u * kConsumerThreads;
            ulonglong2 e = make_ulonglong2(~0ull, 0ull);
            if (i < n_nz) e = __ldcg(nzl + i);
            pk[u] = e.x;
            pc[u] = e.y;
        }
        if (tid == 0) {
            if (n_own > 0) issue(kv[0].x, 0);
            if (n_own > 1) issue(kv[1].x, 1);
        }
#if defined(ARCV_TRACE) && ARCV_TRACE
        if (tid == 0 && pk[0] != 1ull) ARCV_STAMP(1, 9);  // waits for the first pool load
#endif
        for (uint32_t j0 = 0; j0 < n_own; j0 += 2) {
            const uint32_t m = n_own - j0 < 2u ? n_own - j0 : 2u;
            uint64_t key[2], tcn[2] = {0, 0}, pre[2] = {0, 0}, tot[2] = {0, 0};
#pragma unroll
            for (int q = 0; q < 2; ++q) {
                if ((uint32_t)q < m) {
                    const ulonglong2 e = j0 == 0 ? kv[q] : __ldcg(nzl + entry_of(j0 + q));
                    key[q] = e.x;
                    tcn[q] = e.y;
                } else {
                    key[q] = ~0ull - 1;
                }
            }
#pragma unroll
            for (int u = 0; u < kPer; ++u)
#pragma unroll
                for (int q = 0; q < 2; ++q)
                    if ((pk[u] >> 40) == (key[q] >> 40)) {
                        tot[q] += pc[u];
                        pre[q] += (pk[u] & kLtMask) < (key[q] & kLtMask) ? pc[u] : 0ull;
                    }
#pragma unroll
            for (int q = 0; q < 2; ++q) {
                pre[q] = warp_sum_u64(pre[q]);
                tot[q] = warp_sum_u64(tot[q]);
            }
            if ((tid & 31) == 0) {
                sh.red[tid >> 5][0] = pre[0];
                sh.red[tid >> 5][1] = pre[1];
                sh.red[tid >> 5][2] = tot[0];
                sh.red[tid >> 5][3] = tot[1];
            }
            consumer_bar();
            uint64_t r[4] = {0, 0, 0, 0};
#pragma unroll
            for (int w = 0; w < kConsumerWarps; ++w)
#pragma unroll
                for (int c = 0; c < 4; ++c) r[c] += sh.red[w][c];
            if (tid == 0) ARCV_STAMP(1, 3);
#if !defined(ARCV_HALF_TILES) || ARCV_HALF_TILES
            bool half = m == 2 && segs[key[0] >> 40].dtype != ARC_U8 && segs[key[1] >> 40].dtype != ARC_U8;
            if (half) {  // not for dense tiles going straight to pinned memory (staged writes)
#pragma unroll
                for (int q = 0; q < 2; ++q) {
                    const Seg &gq = segs[key[q] >> 40];
                    if (tcn[q] > kStagedMin &&
                        direct_route(gq.report_alias != nullptr, gq.flags, __ldcg(&p.acc[gq.acc_slot].count),
                                     gq.max_report, gq.alias_cap, true))
                        half = false;
                }
            }
            if (half) {
                // the CTA's two tiles at once: warps 0-3 take entry j0 (stage 0),
                // warps 4-7 entry j0 + 1 (stage 1)
                const int grp = tid >> 7, gt = tid & 127;
                const uint64_t kq = grp ? key[1] : key[0];
                const Seg &g = segs[kq >> 40];
                const uint64_t seg_tot = grp ? r[3] : r[2];
                const uint64_t region_cnt = __ldcg(&p.acc[g.acc_slot].count);
                const uint64_t base = (g.flags & kSegBaseFromAcc) ? region_cnt - seg_tot : 0ull;
                const uint64_t excl = base + (grp ? r[1] : r[0]);
                if (gt == 0) p.tile_cnt[g.slot_begin + (kq & kLtMask)] = 0u;  // clean for the next call
                const bool direct = direct_route(g.report_alias != nullptr, g.flags, region_cnt, g.max_report,
                                                 g.alias_cap, true);
                StageInfo si;
                uintptr_t ao, ar;
                uint32_t nbo, nbr;
                plan_tile(g, kq & kLtMask, si, ao, nbo, ar, nbr);
                mbar_wait(&sh.bar[grp], (phase >> grp) & 1u);
                phase ^= 3u;  // both stages' phases complete (each half waits for its own)
                if (excl < g.max_report)  // uniform within the half
                    emit_half_any(g, si, smem + (size_t)grp * kStageBytes, excl | (direct ? kDirectBit : 0ull),
                                  sh.hw[grp], gt, grp);
                consumer_bar();  // both stages and sh.red are free again
                if (tid == 0) {
                    if (j0 + 2 < n_own) issue(__ldcg(p.nz_list + 2 * entry_of(j0 + 2)), 0);
                    if (j0 + 3 < n_own) issue(__ldcg(p.nz_list + 2 * entry_of(j0 + 3)), 1);
                }
                continue;
            }
#endif
#pragma unroll
            for (int q = 0; q < 2; ++q) {
                if ((uint32_t)q >= m) break;
                const uint32_t j = j0 + q;
                const Seg &g = segs[key[q] >> 40];
                const uint64_t seg_tot = r[2 + q];
                uint64_t base = 0;
                if (g.flags & kSegBaseFromAcc) base = __ldcg(&p.acc[g.acc_slot].count) - seg_tot;
                if (tid == 0) p.tile_cnt[g.slot_begin + (key[q] & kLtMask)] = 0u;  // clean for the next call
                emit(key[q], base + r[q], q, true, tcn[q], j == 0);  // ends with a barrier
                if (tid == 0 && j == 1) ARCV_STAMP(1, 10);
                if (tid == 0 && j + 2 < n_own) issue(__ldcg(p.nz_list + 2 * entry_of(j + 2)), q);
            }
        }
        if (tid == 0) ARCV_STAMP(1, 6);
#if defined(ARCV_TAIL_REPS)
      }
#endif
    } else {
        // ------------------------------------------------------ group path
        for (uint32_t sgi = 0; sgi < p.n_segs; ++sgi) {
            const Seg &g = segs[sgi];
            if (g.max_report == 0 || g.n == 0) continue;
            const uint64_t ntiles = (g.n + tile_elems(g.dtype) - 1) / tile_elems(g.dtype);
            const uint64_t ngroups = (ntiles + kGroupTiles - 1) / kGroupTiles;
            const uint32_t *gc = p.group_cnt + g.group_begin;
            uint64_t tot = 0;
            for (uint64_t k = tid; k < ngroups; k += kConsumerThreads) tot += __ldcg(gc + k);
            uint64_t total;
            block_excl_scan(tot, sh.w, &total, tid);
            if (total == 0) continue;  // uniform: nothing to report or to clear
            uint64_t base = 0;
            if (g.flags & kSegBaseFromAcc) base = __ldcg(&p.acc[g.acc_slot].count) - total;

            uint64_t run = base, ord_run = 0;
            for (uint64_t c0 = 0; c0 < ngroups; c0 += kGroupTiles) {
                const uint64_t gi = c0 + tid;
                const uint32_t cnt = gi < ngroups ? __ldcg(gc + gi) : 0u;
                // pack (nonzero ordinal, count): group counts < 2^23, 256 of them < 2^31
                const uint64_t v = ((uint64_t)(cnt != 0) << 40) | cnt;
                uint64_t ctot;
                const uint64_t ex = block_excl_scan(v, sh.w, &ctot, tid);
                const uint64_t gpre = run + (ex & ((1ull << 40) - 1));
                const uint64_t ord = ord_run + (ex >> 40);
                if (tid == 0) sh.n = 0;
                consumer_bar();
                if (cnt != 0 && (ord % G) == b) {
                    const uint32_t k = atomicAdd(&sh.n, 1u);
                    sh.owned[k] = (uint32_t)gi;
                    sh.owned_pre[k] = gpre;
                }
                consumer_bar();
                const uint32_t n_owned = sh.n;
                run += ctot & ((1ull << 40) - 1);
                ord_run += ctot >> 40;
                for (uint32_t q = 0; q < n_owned; ++q) {
                    const uint64_t t0 = (uint64_t)sh.owned[q] * kGroupTiles;
                    const uint64_t gp = sh.owned_pre[q];
                    const uint64_t tg = ntiles - t0 < (uint64_t)kGroupTiles ? ntiles - t0 : (uint64_t)kGroupTiles;
                    uint32_t *tc = p.tile_cnt + g.slot_begin + t0;
                    const uint32_t tcnt = (uint64_t)tid < tg ? __ldcg(tc + tid) : 0u;
                    if (gp < g.max_report) {  // uniform
                        uint64_t gtot;
                        const uint64_t tpre = gp + block_excl_scan(tcnt, sh.w, &gtot, tid);
                        if (tcnt != 0 && tpre < g.max_report) {
                            const uint32_t k = atomicAdd(p.active_cnt, 1u);
                            p.active[2 * k] = ((uint64_t)sgi << 40) | (t0 + tid);
                            p.active[2 * k + 1] = tpre;
                        }
                    }
                    if (tcnt != 0) tc[tid] = 0u;  // clean for the next call
                }
                consumer_bar();
            }
        }
        if (tid == 0) ARCV_STAMP(1, 3);  // group scan done (trace: "prefixes reduced")
        grid_barrier(p.gbar, p.gbar_base, tid);
        if (tid == 0) ARCV_STAMP(1, 9);  // active list complete (trace: "pool loaded")
        const uint32_t n_act = *(volatile uint32_t *)p.active_cnt;
        const uint32_t mine = n_act > b ? (n_act - b + G - 1) / G : 0u;
        if (mine > 0 && tid == 0) issue(__ldcg(p.active + 2 * b), 0);
        for (uint32_t j = 0; j < mine; ++j) {
            const int st = (int)(j & 1);
            if (j + 1 < mine && tid == 0) issue(__ldcg(p.active + 2 * (b + (j + 1) * G)), st ^ 1);  // prefetch
            const uint64_t key = __ldcg(p.active + 2 * (b + j * G));
            const uint64_t excl = __ldcg(p.active + 2 * (b + j * G) + 1);
            emit(key, excl, st, false, 0, j == 0);
        }
        if (tid == 0) ARCV_STAMP(1, 6);
    }
    // Report entries in pinned host memory need no system-scope fence here:
    // this CTA's gpu-scope release (fence + done counter) is acquired by the
    // last CTA, whose fence.acq_rel.sys before the completion word is
    // cumulative -- every write that happens-before it (these entries
    // included) is visible to the host that acquires the word.  One PCIe
    // flush per call instead of one per writing CTA.
    // (-DARCV_WRITER_SYS=1: a system-scope fence in every writing CTA.)
#if defined(ARCV_WRITER_SYS) && ARCV_WRITER_SYS
    const bool wrote_host = p.report_host != 0 || sh.wrote != 0;
#else
    const bool wrote_host = false;
#endif
    if (p.finalize) {
        const bool last = last_cta(p, tid, kConsumerThreads, &sh.last, wrote_host, done_base);
        if (tid == 0) ARCV_STAMP(1, 11);
        // a report kept in device memory (the caller's buffer or HBM staging that
        // the host copies later, stream-ordered) needs no system fence before the
        // completion word: the slots validate themselves (slot_tag)
        if (last && !(k1_published_if_empty && n_nz == 0))
            publish(p, tid, kConsumerThreads, p.report_host != 0, n_nz, have_pre ? &pre_acc : nullptr);
        if constexpr (XF) {
            if (p.xfused) exchange_tail(p, tid, last, smem);
        }
    }
    if (tid == 0) ARCV_STAMP(1, 7);
}

// K2: the report phase as its own launch (cooperative: the group path has a
// grid barrier), a programmatic dependent of K1.  Used when the fused tail does
// not fit K1's stage memory (fewer than 3 stages) or ARCV_FUSED=0.
// grid: SMs x co-resident CTAs; block: 256; dynamic smem: kReportSmem.
template <int NSEG>
__global__ void __launch_bounds__(kConsumerThreads) arcv_compact_kernel(const __grid_constant__ ParamsN<NSEG> pn) {
    extern __shared__ __align__(128) uint8_t smem[];
    const Params &p = pn;
    const Seg *segs = p.segs ? p.segs : pn.inline_segs;
    if (threadIdx.x == 0) ARCV_STAMP(1, 0);
    // wait for K1's completion (and the visibility of its writes) before
    // touching any of them
    asm volatile("griddepcontrol.wait;" ::: "memory");
    asm volatile("griddepcontrol.launch_dependents;" ::: "memory");  // the exchange kernel, if any
    report_phase<false>(p, segs, smem, (int)threadIdx.x, p.done_base, true);
}


// ------------------------------------------------------------------ K1: stream
// XF: the sharded exchange is fused into this kernel's tail (its own
// instantiation, so single-GPU calls carry none of the exchange code).
// Per-tile bookkeeping for the report phase (ARCV_PRODUCER_BOOKKEEP): the
// consumer warps add their counts to the stage's shared word with fire-and-
// forget shared-memory reductions before releasing the stage; the producer
// lane, when the stage comes back empty, reads the word (released by the
// mbarrier), adds a nonzero count to the tile and group counters and -- while
// the pool has room -- lists the tile, then clears the word before the refill.
// The consumers' loop thus carries no atomics with a return value and no
// global memory round trip (a dense call streamed ~3.5 % slower with them).  A tile left out must leave the
// pool count ABOVE kPoolCap: a count of exactly kPoolCap means "all listed",
// so a tile that finds it full lifts it to kPoolCap + 1; once the producer has
// seen the count at or past kPoolCap it stops reading it (`pool_full`).
__device__ __forceinline__ void producer_bookkeep(const Params &p, const Seg *segs, const StageInfo &si,
                                                  uint32_t *tc_word, bool &pool_full) {
    const uint32_t tc = *tc_word;  // the consumer warps' counts (shared-memory reductions)
    if (tc == 0) return;
    *tc_word = 0u;  // before the stage is refilled
    const Seg &g = segs[si.seg];
    const uint64_t lt = si.tile - g.tile_begin;
    atomicAdd(p.tile_cnt + g.slot_begin + lt, tc);
    atomicAdd(p.group_cnt + g.group_begin + lt / kGroupTiles, tc);
    if (pool_full) return;
    const uint32_t v = *(volatile uint32_t *)p.nz_cnt;
    if (v < (uint32_t)kPoolCap) {
        const uint32_t k = atomicAdd(p.nz_cnt, 1u);
        if (k < (uint32_t)kPoolCap) {
            p.nz_list[2 * k] = ((uint64_t)si.seg << 40) | lt;
            p.nz_list[2 * k + 1] = tc;
        } else {
            pool_full = true;  // the count is now above kPoolCap
        }
    } else {
        if (v == (uint32_t)kPoolCap) atomicMax(p.nz_cnt, (uint32_t)kPoolCap + 1u);
        pool_full = true;
    }
}
constexpr int kProdBar = 5;  // named barrier: consumers wait for the producer's last bookkeeping

template <int S, int MINB, int NSEG, bool XF = false, int DTM = kAllDtypes>
__global__ void __launch_bounds__(kThreads, MINB) arcv_stream_kernel(const __grid_constant__ ParamsN<NSEG> pn) {
    const Params &p = pn;
    extern __shared__ __align__(128) uint8_t smem[];
    __shared__ __align__(8) uint64_t full_bar[S];
    __shared__ __align__(8) uint64_t empty_bar[S];
    __shared__ StageInfo info[S];
    __shared__ uint64_t s_red_u[kConsumerWarps][2];
    __shared__ double s_red_d[kConsumerWarps][2];
    __shared__ int s_last;
    __shared__ uint32_t s_tile[S];
#if ARCV_PRODUCER_BOOKKEEP
    __shared__ uint32_t s_tc[S];  // per stage: the tile's mismatch count (reporting regions)
#endif

    const Seg *segs = p.segs ? p.segs : pn.inline_segs;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;

    if (threadIdx.x == 0) {
        for (int s = 0; s < S; ++s) {
            s_tile[s] = 0u;
#if ARCV_PRODUCER_BOOKKEEP
            s_tc[s] = 0u;
#endif
            mbar_init(&full_bar[s], 1);
            mbar_init(&empty_bar[s], kConsumerWarps);
        }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();

    // ------------------------------------------------------------ producer
    if (warp == 0) {
        if (lane == 0) {
            const uint64_t policy = evict_first_policy();
            uint64_t t = 0, t_end = 0;  // current run [t, t_end)
#if ARCV_PRODUCER_BOOKKEEP
            bool pool_full = false;
#endif
            for (uint32_t i = 0;; ++i, ++t) {
                const int s = i % S;
                if (i >= (uint32_t)S) {
                    mbar_wait(&empty_bar[s], ((i / S) - 1) & 1);
#if ARCV_PRODUCER_BOOKKEEP
                    if (p.k2) producer_bookkeep(p, segs, info[s], &s_tc[s], pool_full);  // the tile it held
#endif
                }
                if (t >= t_end) {
#if ARCV_GUIDED
                  if (p.guided) {
                    // the counter ends at exactly base + total_tiles: a run that
                    // crosses the end gives its overshoot back, a run past the
                    // end all of it (the counter never drops below the end)
                    // size the run from the counter's current value (a stale
                    // estimate could hand a long run out near the end)
                    const uint64_t cur = *(volatile unsigned long long *)p.ticket - p.ticket_base;
                    const uint64_t rem = p.total_tiles > cur ? p.total_tiles - cur : 0;
                    uint64_t c = rem / (kGuide * gridDim.x);
                    c = c < 1 ? 1 : (c > kChunkMax ? kChunkMax : c);
                    const uint64_t old = atomicAdd(p.ticket, (unsigned long long)c) - p.ticket_base;
                    if (old >= p.total_tiles) {
                        atomicAdd(p.ticket, (unsigned long long)(0ull - c));
                        t = p.total_tiles;
                    } else {
                        if (old + c > p.total_tiles)
                            atomicAdd(p.ticket, (unsigned long long)(0ull - (old + c - p.total_tiles)));
                        t = old;
                        t_end = old + c < p.total_tiles ? old + c : p.total_tiles;
                    }
                  } else
#endif
                  {
                    t = atomicAdd(p.ticket, 1ull) - p.ticket_base;
                    t_end = t + 1;
                  }
                }
                if (t >= p.total_tiles) {
                    info[s].tile = ~0ull;
                    mbar_arrive(&full_bar[s]);
#if ARCV_PRODUCER_BOOKKEEP
                    // the tiles still with the consumers: iterations i - S + 1 .. i - 1
                    if (p.k2)
                        for (uint32_t j = i >= (uint32_t)(S - 1) ? i - (S - 1) : 0u; j < i; ++j) {
                            mbar_wait(&empty_bar[j % S], (j / S) & 1);
                            producer_bookkeep(p, segs, info[j % S], &s_tc[j % S], pool_full);
                        }
#endif
                    break;
                }
                const uint32_t sg = find_seg(segs, p.n_segs, t);
                const Seg &g = segs[sg];
                StageInfo &si = info[s];
                uintptr_t ao, ar;
                uint32_t nbo, nbr;
                plan_tile(g, t - g.tile_begin, si, ao, nbo, ar, nbr);
                si.tile = t;
                si.seg = sg;
                uint8_t *dst = smem + (size_t)s * kStageBytes;
                mbar_arrive_expect_tx(&full_bar[s], nbo + nbr);
                bulk_g2s(dst, reinterpret_cast<const void *>(ao), nbo, &full_bar[s], policy);
                bulk_g2s(dst + kStageArrayBytes, reinterpret_cast<const void *>(ar), nbr, &full_bar[s], policy);
            }
        }
#if ARCV_PRODUCER_BOOKKEEP
        if (p.k2) {  // the bookkeeping is complete before any consumer arrives at the grid barrier
            // (bar.arrive orders the lane's global writes for the consumers, whose
            // gpu-scope release before the done count then covers them)
            __syncwarp();
            asm volatile("bar.arrive %0, %1;" ::"n"(kProdBar), "n"(kConsumerThreads + 32) : "memory");
        }
#endif
        return;
    }

    // ------------------------------------------------------------ consumers
    const int ctid = threadIdx.x - 32;
    // zero the other parity's group counters and active-list length for the next
    // launch (the previous launch that used them has completed: same stream)
    if (blockIdx.x == 0 && ctid == 0 && p.active_cnt_zero) {
        *p.active_cnt_zero = 0u;
        *p.nz_cnt_zero = 0u;
    }
    for (uint64_t k = (uint64_t)blockIdx.x * kConsumerThreads + ctid; k < p.n_group_zero;
         k += (uint64_t)gridDim.x * kConsumerThreads)
        p.group_zero[k] = 0;

    ThreadAcc acc;
    acc.reset();
    int cur = -1;
    SegHot g;
    if (ctid == 0) ARCV_STAMP(0, 0);
    for (uint32_t i = 0;; ++i) {
        const int s = i % S;
        mbar_wait(&full_bar[s], (i / S) & 1);
        if (ctid == 0 && i == 0) ARCV_STAMP(0, 4);
        const StageInfo si = info[s];
        if (si.tile == ~0ull) break;
        if ((int)si.seg != cur) {
#if defined(ARCV_TRACE) && ARCV_TRACE
            if (ctid == 0 && si.seg < 16 && g_trace[2][blockIdx.x < (unsigned)kTraceCtas ? blockIdx.x : 0][2 * si.seg] == 0)
                ARCV_STAMP(2, 2 * si.seg);
#endif
            const uint32_t slot = segs[si.seg].acc_slot;
            if (cur >= 0 && slot != g.acc_slot) flush_acc(p.acc, g.acc_slot, g.dtype, acc, ctid, s_red_u, s_red_d);
            cur = (int)si.seg;
            g.load(segs[si.seg]);
            g.seed_sh = s_red_d;
        }
        const uint8_t *so = smem + (size_t)s * kStageBytes;
        const uint32_t cnt = (p.flags & kFlagProbe) ? 0u : eval_any<DTM>(so, so + kStageArrayBytes, si, ctid, g, acc);
        acc.count += cnt;
        if (ctid == 0 && i == 0) ARCV_STAMP(0, 5);
#if defined(ARCV_TRACE) && ARCV_TRACE
        if (ctid == 0 && si.seg < 16 && g_trace[2][blockIdx.x < (unsigned)kTraceCtas ? blockIdx.x : 0][2 * si.seg + 1] == 0)
            ARCV_STAMP(2, 2 * si.seg + 1);
#endif
#if ARCV_PRODUCER_BOOKKEEP
        if (g.max_report != 0) {
            // this warp's share of the tile's count, for the producer's bookkeeping
            // (read once the stage's empty barrier completes)
            const uint32_t wc = __reduce_add_sync(0xffffffffu, cnt);
            if (lane == 0 && wc != 0u)
                asm volatile("red.shared.add.u32 [%0], %1;" ::"r"(smem_u32(&s_tc[s])), "r"(wc) : "memory");
        }
#else
        if (g.max_report != 0) {
            // Per-tile count for the report phase: warps fold their counts into the stage's
            // shared word (arrivals << 24 | count); the last warp publishes the
            // tile (2 global atomics per tile with mismatches, none otherwise)
            // and clears the word before the stage can be reused.
            const uint32_t wc = __reduce_add_sync(0xffffffffu, cnt);
            if (lane == 0) {
                const uint32_t old = atomicAdd(&s_tile[s], (1u << 24) | wc);
                if ((old >> 24) == kConsumerWarps - 1) {
                    const uint32_t tc = (old & 0xffffffu) + wc;
                    s_tile[s] = 0u;
                    if (tc != 0) {
                        const uint64_t lt = si.tile - g.tile_begin;
                        atomicAdd(p.tile_cnt + g.slot_begin + lt, tc);
                        atomicAdd(p.group_cnt + g.group_begin + lt / kGroupTiles, tc);
                        // short list of nonzero tiles for the pool path (checked
                        // before the atomic so a dense call stops touching it).
                        // A tile left out must leave the count ABOVE kPoolCap:
                        // a count of exactly kPoolCap means "all listed", so a
                        // tile that finds the list full lifts it to kPoolCap + 1
                        // (without this, 2049 nonzero tiles could end with a
                        // count of 2048 and take the pool path one tile short).
                        // (Round 2 measured doing this after the stage release,
                        // with a per-CTA "pool full" flag: C5 -1 %, C4 +2.2 %,
                        // profiles/r02s4_ab_late_tile_publish_rejected.log.)
                        const uint32_t v = *(volatile uint32_t *)p.nz_cnt;
                        if (v < (uint32_t)kPoolCap) {
                            const uint32_t k = atomicAdd(p.nz_cnt, 1u);
                            if (k < (uint32_t)kPoolCap) {
                                p.nz_list[2 * k] = ((uint64_t)si.seg << 40) | lt;
                                p.nz_list[2 * k + 1] = tc;
                            }
                        } else if (v == (uint32_t)kPoolCap) {
                            atomicMax(p.nz_cnt, (uint32_t)kPoolCap + 1u);
                        }
                    }
                }
            }
        }
#endif
        if (p.flags & 1u) asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
        __syncwarp();
        if (lane == 0) mbar_arrive(&empty_bar[s]);  // stage may be refilled now
    }
#if ARCV_PRODUCER_BOOKKEEP
    if (p.k2) asm volatile("bar.sync %0, %1;" ::"n"(kProdBar), "n"(kConsumerThreads + 32) : "memory");
#endif
    // A dependent launch (exchange kernel or K2, PDL) may be scheduled from here on; it
    // waits for this grid's completion before reading anything it wrote.
    if (ctid == 0) ARCV_STAMP(0, 1);
    asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
    if (cur >= 0) flush_acc(p.acc, g.acc_slot, g.dtype, acc, ctid, s_red_u, s_red_d);
    if (ctid == 0) ARCV_STAMP(0, 2);
    if constexpr (S * kStageBytes >= kReportSmem) {
        if (p.fused) {
            // Fused report phase (cooperative launch: every CTA is resident).
            // Grid barrier on the done counter: the tile counts and the pool
            // are complete once every CTA has flushed.  The stage memory is
            // free (the sentinel stage follows every real fill).
            if (ctid == 0) {
                ARCV_STAMP(1, 0);
                fence_gpu();
                const unsigned long long prev = atomicAdd(p.done, 1ull);
                s_last = (prev - p.done_base) == (unsigned long long)(gridDim.x - 1);
                if (!s_last)
                    while (ld_acquire_u64(p.done) - p.done_base < (unsigned long long)gridDim.x) __nanosleep(32);
            }
            consumer_bar();
            // The CTA that arrives last has seen every count: with no tile to
            // report (the common, clean call) the results are final now, so it
            // publishes at once, and no CTA runs the report phase -- each only
            // keeps its counter contract (one grid-barrier arrival, and with
            // `finalize` one done arrival) with fire-and-forget reductions.
            const uint32_t n_nz = *(volatile uint32_t *)p.nz_cnt;  // final: every CTA has arrived
            if (n_nz == 0u) {
                if (s_last && p.finalize) publish(p, ctid, kConsumerThreads, false, 0u);  // no entry written anywhere
                if (ctid == 0) {
                    asm volatile("red.relaxed.gpu.global.add.u64 [%0], 1;" ::"l"(p.gbar) : "memory");
                    if (p.finalize) asm volatile("red.relaxed.gpu.global.add.u64 [%0], 1;" ::"l"(p.done) : "memory");
                }
                if constexpr (XF) {
                    if (p.xfused) exchange_tail(p, ctid, s_last != 0, smem);  // the leader published the mirror
                }
                return;
            }
            report_phase<XF>(p, segs, smem, ctid, p.done_base + gridDim.x, true, n_nz);
            return;
        }
    }
    // Unfused (K2 follows): the last CTA publishes at once unless K2 has report
    // entries to write: with no mismatch in any reporting region the host wakes
    // here while K2 -- then a no-op -- runs in the background.
    if ((p.finalize || p.k2) && last_cta(p, ctid, kConsumerThreads, &s_last, false, p.done_base)) {
        fence_gpu();
        if (p.finalize && (!p.k2 || *(volatile uint32_t *)p.nz_cnt == 0u))
            publish(p, ctid, kConsumerThreads, false);  // count-only / clean: no report entry written
    }
    if constexpr (XF) {
        if (p.xfused) exchange_tail(p, ctid, s_last != 0, smem);  // count-only sharded call (no K2 then)
    }
    if (ctid == 0) ARCV_STAMP(0, 3);
}


}  // namespace arcv
