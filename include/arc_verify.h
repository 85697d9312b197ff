/*
 * arc_verify.h -- C ABI of the B200-native kernel-verification result comparison.
 *
 * The operation (PAPER.md = /root/reference/PAPER.md, cited as P:<line>):
 *   sec. III-A, P:159  "we propose to compare these results at the granularity of
 *                       a GPU kernel": the outputs of a translated GPU region are
 *                       compared with the outputs of the sequential CPU region.
 *   sec. III-A, P:171  "all data modified by the kernel are copied back to a
 *                       temporary space on the CPU after the kernel finished";
 *                       Listing 2 line 11: "Result comparison codes
 *                       will be added" after "#pragma acc wait(1)".
 *   sec. III-A, P:199  "If the output difference is bigger than the allowed error
 *                       margin, then an error will be reported to the user ...
 *                       the transformation allows users to configure the error
 *                       margin".
 *   sec. III-A, P:161  the margin exists because "CPU and GPU may use different
 *                       numbers of bits to store floating-point numbers, and
 *                       non-deterministic computation order".
 * This library runs the comparison itself on the GPU (the paper ran it on the
 * host CPU over data copied back over PCIe), so only the
 * summary and the report cross to the host.
 *
 * Per element i, for float dtypes (x = (double)out[i], y = (double)ref[i],
 * exact widening; arithmetic in IEEE fp64, round-to-nearest, no FMA contraction,
 * no flush-to-zero):
 *   rule 1  x == y                -> match, d = 0, r = 0        (covers +-0, equal Inf)
 *   rule 2  isnan(x) && isnan(y)  -> match, d and r excluded from the maxima
 *   rule 3  isnan(x) || isnan(y)  -> mismatch, d and r excluded
 *   rule 4  isinf(y)              -> mismatch, d = r = +Inf
 *   rule 5  d = |x - y|, t = abs_tol + (rel_tol * |y|) as two rounded operations;
 *           match iff d <= t; r = d / |y| (+Inf if d = +Inf or y = 0)
 * For integer dtypes: match iff out[i] == ref[i] (tolerances ignored);
 * d = |out[i] - ref[i]| computed exactly and converted to double (RN); no r.
 * The readings behind rules 1-5 (the paper gives no formula) are DESIGN.md
 * sec. 3, R1-R12.
 *
 * Result: n_mismatch = exact count; max_abs_err / max_rel_err = max of the
 * defined d / r (0 if none; max_rel_err = 0 for integers); report = the first
 * max_report mismatches in ascending index order, each (index, raw bits of
 * out[i], raw bits of ref[i]) zero-extended to 64 bits.  The GPU result is
 * bit-identical to the CPU oracle (oracle/arc_oracle.c) for any launch geometry,
 * batching or sharding.
 *
 * Conventions
 *  - Every call returns an arc_status_t.  A mismatch is data, not an error
 *    (ARC_OK with n_mismatch > 0).
 *  - One context per process; calls are not thread-safe (the caller serialises).
 *  - Work is enqueued on the stream given at init (or arc_verify_set_stream) and
 *    every call returns after its result is on the host (the paper's
 *    "acc wait" before comparison, Listing 2 line 10).
 *  - Ownership: the library never owns or frees caller arrays or report
 *    buffers; it owns its workspace (look-back status words, accumulators,
 *    staging), allocated lazily, grown on demand, freed by arc_verify_finalize.
 */
#ifndef ARC_VERIFY_H
#define ARC_VERIFY_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
    ARC_OK = 0,
    ARC_E_INVAL = -1,       /* bad argument (see each call)                        */
    ARC_E_NOINIT = -2,      /* called before arc_verify_init                       */
    ARC_E_CUDA = -3,        /* a CUDA runtime call failed (text: arc_verify_last_error) */
    ARC_E_NCCL = -4,        /* an NCCL call failed, or NCCL could not be loaded    */
    ARC_E_NOMEM = -5,       /* workspace allocation failed                         */
    ARC_E_UNSUPPORTED = -6  /* valid request this build does not support           */
} arc_status_t;

typedef enum { ARC_F32 = 0, ARC_F64 = 1, ARC_I32 = 2, ARC_I64 = 3, ARC_U8 = 4 } arc_dtype_t;

/* One reported mismatch: 24 bytes, raw bit patterns zero-extended. */
typedef struct {
    uint64_t index;    /* element index (global index when sharded)  */
    uint64_t out_bits; /* raw bits of out[index]                     */
    uint64_t ref_bits; /* raw bits of ref[index]                     */
} arc_mismatch_t;

typedef struct {
    uint64_t n;             /* elements compared (global n when sharded)            */
    uint64_t n_mismatch;    /* exact number of mismatches                           */
    double max_abs_err;     /* max defined d; 0 for empty / all-NaN                 */
    double max_rel_err;     /* max defined r; 0 for integer dtypes                  */
    uint64_t n_reported;    /* = min(n_mismatch, max_report)                        */
    arc_mismatch_t *report; /* CALLER-owned, capacity >= min(max_report, n) entries
                               (sharded: the GLOBAL n);
                               host memory (pageable or pinned) or device memory on
                               the library's device (then nothing crosses PCIe)     */
} arc_verify_result_t;

typedef struct {
    int device;                 /* CUDA device ordinal                                    */
    void *stream;               /* cudaStream_t to enqueue on; NULL = a library-owned
                                   non-blocking stream (the caller orders its own work);
                                   (void*)1 = cudaStreamLegacy, the legacy default stream */
    int rank, nranks;           /* sharded mode when nranks > 1                           */
    const void *nccl_unique_id; /* 128-byte ncclUniqueId (same on all ranks), or NULL.
                                   nranks > 1 needs it, or the peer windows
                                   (arc_verify_peer_export / _open), or both; with
                                   nranks == 1 an id selects the collective path over a
                                   1-rank communicator                                    */
} arc_verify_opts_t;

/*
 * Optional per-region checks (sec. III-A and III-C; NEXT row N2; DESIGN.md
 * readings R10, R11).  flags = 0 disables both.
 *   ARC_CHECK_MIN_VALUE  ("minValueToCheck": "result is compared only if
 *       its value is bigger than a specified threshold"): element i is not
 *       compared when |ref[i]| <= min_value -- it is a match and its d, r are
 *       excluded from the maxima.  A NaN ref is still compared.
 *   ARC_CHECK_VALUE_BOUNDS (value-bound directives: differences that "fall
 *       within the user-specified bound" are ignored): a mismatch with
 *       lo <= out[i] <= hi is ignored -- a match, d and r excluded.
 * Integer values enter both checks as (double)value, rounded to nearest.
 * Errors: ARC_E_INVAL for unknown flag bits or NaN min_value / lo / hi.
 */
enum { ARC_CHECK_MIN_VALUE = 1u, ARC_CHECK_VALUE_BOUNDS = 2u };
typedef struct {
    uint32_t flags;
    double min_value;
    double lo, hi;
} arc_verify_check_t;

typedef struct {
    const void *out;  /* region output computed by the GPU kernel                  */
    const void *ref;  /* sequential reference output                               */
    uint64_t n;       /* elements (row-major flattened)                            */
    arc_dtype_t dtype;
    double abs_tol, rel_tol;
    uint64_t max_report;
    const char *name; /* for printing only; may be NULL                            */
    const arc_verify_check_t *check; /* optional checks (N2); NULL = none            */
} arc_verify_region_t;

/*
 * arc_verify_init -- create the process context.
 *   opts == NULL: device 0, library-owned stream, one rank.
 *   nranks > 1: sharded mode.  The exchange runs over the peer windows when
 *   they are open (arc_verify_peer_export + arc_verify_peer_open, below), else
 *   over NCCL: nccl_unique_id is then the id produced by
 *   arc_verify_get_unique_id on one rank and shared with all ranks, and NCCL
 *   (libnccl.so.2, the one already loaded by the process if any) is opened at
 *   run time.
 * Errors: ARC_E_INVAL (bad device / rank / nranks), ARC_E_CUDA, ARC_E_NCCL.
 * Calling init twice without finalize returns ARC_E_INVAL.
 */
int arc_verify_init(const arc_verify_opts_t *opts);

/*
 * arc_verify_compare -- verify one region: out[0..n) against ref[0..n).
 *   out, ref : device pointers on the library's device, OR host pointers
 *              (pinned or pageable); host inputs are streamed to the device in
 *              chunks that overlap the comparison (the paper's data flow, where
 *              the sequential reference lives in host memory).
 *              Each pointer must be aligned to the element size.
 *   n        : elements; n == 0 is legal (all-zero result).
 *   dtype    : element type of both arrays.
 *   abs_tol, rel_tol : finite and >= 0 (ignored for integer dtypes).
 *   max_report : report capacity / truncation; 0 = count only.
 *   result   : caller-owned; result->report must hold min(max_report, n)
 *              entries when max_report > 0.
 * Sharded mode (nranks > 1): COLLECTIVE -- every rank calls it with the same
 * dtype, tolerances and max_report; out/ref/n are the rank's contiguous shard;
 * global index = sum of n over lower ranks + local index; every rank receives
 * the identical global result.
 * Errors: ARC_E_INVAL (NULL arrays with n > 0, unknown dtype, NaN / negative /
 * infinite tolerance, NULL result, NULL report with max_report > 0, misaligned
 * pointer, device pointer on another device), ARC_E_NOINIT, ARC_E_CUDA,
 * ARC_E_NCCL, ARC_E_NOMEM.  ARC_E_CUDA is also returned when the kernels
 * finished without publishing this call's results ("completion word
 * missing"): the library never returns a previous call's numbers as ARC_OK.
 */
int arc_verify_compare(const void *out, const void *ref, uint64_t n, arc_dtype_t dtype,
                       double abs_tol, double rel_tol, uint64_t max_report,
                       arc_verify_result_t *result);

/*
 * arc_verify_compare_ex -- arc_verify_compare with the optional checks of
 * arc_verify_check_t (check may be NULL).  Not collective in sharded mode
 * unless check is NULL (the checks are then applied locally on each rank).
 */
int arc_verify_compare_ex(const void *out, const void *ref, uint64_t n, arc_dtype_t dtype,
                          double abs_tol, double rel_tol, uint64_t max_report,
                          const arc_verify_check_t *check, arc_verify_result_t *result);

/*
 * arc_verify_batch -- verify n_regions regions ("all data written by the kernels
 * are examined") in ONE grid when all inputs are device-resident.
 * results[k] equals what arc_verify_compare would return for regions[k] alone.
 * Same argument rules as arc_verify_compare, per region.  Not collective: in
 * sharded mode the batch is verified locally on each rank.
 */
int arc_verify_batch(const arc_verify_region_t *regions, size_t n_regions,
                     arc_verify_result_t *results);

/* Release the workspace, the NCCL communicator and the owned stream. */
int arc_verify_finalize(void);

/* Static text for a status code. */
const char *arc_verify_strerror(int status);

/* Text of the last failing CUDA/NCCL call in this process (static buffer). */
const char *arc_verify_last_error(void);

/* Enqueue subsequent work on `stream` (cudaStream_t on the library's device). */
int arc_verify_set_stream(void *stream);

/* Fill `id` (128 bytes) with a fresh ncclUniqueId for sharded init.
 * Errors: ARC_E_NCCL if NCCL cannot be loaded. */
int arc_verify_get_unique_id(void *id);

/*
 * Kernel timing for benchmarks: when enabled, the library records CUDA events
 * on its stream around every compare-kernel launch and accumulates the launch
 * count and total device time (ms) until arc_verify_kernel_stats(..., reset=1).
 */
int arc_verify_set_timing(int enable);
int arc_verify_kernel_stats(uint64_t *launches, double *total_ms, int reset);

/* Number of the library's kernels launched since arc_verify_init (every kernel:
 * compare, compact, merge / exchange, checksum); 0 before init.  Benchmarks
 * report it as their launch count. */
uint64_t arc_verify_launch_count(void);

/*
 * arc_verify_probe_read -- DIAGNOSTIC (benchmarks only, not part of the method):
 * stream two device buffers of `bytes` each through the same bulk-copy pipeline
 * as the comparison, with the predicate disabled, `iters` times, and return the
 * achieved read bandwidth in GB/s (2 * bytes * iters / time).  It is the in-run
 * read-only ceiling the comparison kernel is judged against.  Each launch is
 * timed on its own from an idle stream (CUDA events around the launch), as a
 * compare call runs and as arc_verify_kernel_stats times it.
 * Errors: ARC_E_INVAL (NULL / host buffers, bytes == 0, iters < 1), ARC_E_NOINIT.
 */
int arc_verify_probe_read(const void *a, const void *b, uint64_t bytes, int iters, double *gbs);

/*
 * arc_verify_checksum -- the debug-assertion checksum screen (sec. III-C, P:291:
 * "performing customized bug detection (e.g., establishing checksums and
 * verifying them)"; NEXT row N4).  `data` is device memory on the library's
 * device (any alignment), `bytes` its length.  out[0] = sum of h_i mod 2^64,
 * out[1] = xor of h_i, where h_i = F(w_i + i * 0x9E3779B97F4A7C15), w_i the
 * little-endian 64-bit words (last one zero-padded) and F the splitmix64
 * finalizer.  Reads one array (half a comparison's bytes); equal checksums of a
 * kernel output and of its reference mean bitwise-identical data with
 * probability 1 - 2^-64 per pair.  Errors: ARC_E_INVAL, ARC_E_NOINIT, ARC_E_CUDA.
 */
int arc_verify_checksum(const void *data, uint64_t bytes, uint64_t out[2]);

/* ------------------------------------------------------------------------
 * Region selection and report printing (NEXT row N3), host-only.
 * Sec. III-A: "a user can specify which specific kernels to verify by
 * adding directives or using environment variables (e.g.,
 * 'verificationOptions=complement=0,kernels=main_kernel0' ...)".  Reading
 * (R20): comma-separated key=value pairs, an optional
 * "verificationOptions=" prefix; `kernels` = region names separated by ':'
 * (further comma tokens without '=' are also names); complement=0 (default)
 * verifies only the listed regions, complement=1 all but them; no `kernels`
 * key selects every region; other keys are ignored.  options == NULL reads the
 * environment variable verificationOptions (then ARC_VERIFICATION_OPTIONS);
 * unset selects every region.
 * ------------------------------------------------------------------------ */

/* 1 if region `name` is selected, 0 if not, ARC_E_INVAL for malformed options. */
int arc_verify_selected(const char *options, const char *name);

/* arc_verify_batch over the selected regions only; selected[k] (may be NULL)
 * receives 1/0; an unselected region's result is zeroed (its report pointer
 * kept).  Errors as arc_verify_batch, plus ARC_E_INVAL for malformed options. */
int arc_verify_batch_selected(const arc_verify_region_t *regions, size_t n_regions, const char *options,
                              arc_verify_result_t *results, uint8_t *selected);

/* Human-readable report of one result ("an error will be reported to the user",
 * P:199): a summary line, then up to max_entries entries "[index] out=.. ref=.."
 * with decoded values and raw bits.  The report may be host or device memory.
 * Writes a NUL-terminated string into buf (truncated to cap - 1 bytes) and
 * returns the full length.  Errors: ARC_E_INVAL, ARC_E_CUDA. */
int arc_verify_format_result(const char *name, arc_dtype_t dtype, double abs_tol, double rel_tol,
                             const arc_verify_result_t *result, uint64_t max_entries, char *buf, size_t cap);

/* ABI version (major << 16 | minor). */
uint32_t arc_verify_version(void);

/* Build description of THIS library (static string, never NULL): the nvcc
 * flags and -D defines it was compiled with, then the compile-time knobs as
 * seen by the code itself, e.g. "nvcc: -gencode ... -fmad=false -ftz=false
 * ...; knobs: ARCV_DIRECT_DYN=4096 ...; defaults=1".  The bit-exact contract
 * depends on -fmad=false -ftz=false -prec-div=true;
 * "defaults=0" marks an A/B variant build.  Needs no GPU and no init. */
const char *arc_verify_build_info(void);

/* ------------------------------------------------------------------------
 * Sharded building blocks (the cross-GPU merge, DESIGN.md sec. 2 step a8).
 * The paper is single-GPU; sharding one large output array across the
 * GPUs of one box is this build's extension.  arc_verify_compare in sharded
 * mode = arc_verify_shard_local -> ncclAllGather of the packets ->
 * arc_verify_shard_merge (+ grouped ncclBroadcast of report entries that do
 * not fit in a packet).  The pieces are exported so a single GPU can run the
 * exact merge path over P simulated shards ("loopback"), and so host code can
 * check the merge plan without a GPU.
 * ------------------------------------------------------------------------ */

/* Per-shard summary header, the first 32 bytes of a packet. */
typedef struct {
    uint64_t n;            /* shard length (elements)            */
    uint64_t n_mismatch;   /* local exact count                  */
    uint64_t max_abs_bits; /* bit pattern of the local max_abs   */
    uint64_t max_rel_bits; /* bit pattern of the local max_rel   */
} arc_shard_header_t;

/* Where rank r's entries land in the global report. */
typedef struct {
    uint64_t index_offset; /* sum of n over lower ranks (global index base)          */
    uint64_t prefix;       /* sum of n_mismatch over lower ranks (report position)   */
    uint64_t contrib;      /* min(n_mismatch_r, max(0, max_report - prefix))         */
} arc_shard_plan_t;

/*
 * arc_verify_merge_plan -- HOST function, needs no GPU and no init.  Given the
 * nranks headers in rank order, fill plan[0..nranks) and the global header
 * (sum of counts and n, max of the max bit patterns -- valid because the
 * values are non-negative doubles).  Errors: ARC_E_INVAL on NULL pointers or
 * nranks < 1.
 */
int arc_verify_merge_plan(const arc_shard_header_t *hdrs, int nranks, uint64_t max_report,
                          arc_shard_plan_t *plan, arc_shard_header_t *global);

/* Bytes of a packet holding `entries` report entries: 32 + 24 * entries. */
size_t arc_verify_packet_bytes(uint64_t entries);

/*
 * arc_verify_shard_local -- compare one local shard (device pointers) and write
 * its packet to packet_dev (device memory of capacity
 * arc_verify_packet_bytes(packet_entries) bytes, caller-owned): header, then
 * the first min(n_mismatch, max_report) local mismatches with LOCAL indices.
 * The kernel may write up to min(max_report, n) entries, so that must not
 * exceed packet_entries: ARC_E_INVAL otherwise (nothing is launched).  Other
 * errors as arc_verify_compare.
 */
int arc_verify_shard_local(const void *out, const void *ref, uint64_t n, arc_dtype_t dtype, double abs_tol,
                           double rel_tol, uint64_t max_report, void *packet_dev, uint64_t packet_entries);

/*
 * arc_verify_shard_merge -- merge nranks gathered packets (device memory,
 * rank r's packet at byte offset r * arc_verify_packet_bytes(packet_entries))
 * into the global result, on the GPU.  result->report as in
 * arc_verify_compare.  Every contribution must fit in its packet
 * (plan.contrib <= packet_entries), else ARC_E_UNSUPPORTED (the collective
 * path then broadcasts the remainder).
 */
int arc_verify_shard_merge(const void *gathered_dev, int nranks, uint64_t packet_entries, uint64_t max_report,
                           arc_verify_result_t *result);

/* ------------------------------------------------------------------------
 * Peer-memory exchange (the B200 path of step a8).
 * Each rank owns a "window" in its HBM -- 2 x 256 flag words and two packets
 * (call parities) of {32-byte header, max_report_cap entries} -- mapped into
 * every other rank through CUDA IPC (NVLink / NVSwitch peer memory).  A
 * sharded arc_verify_compare with max_report <= max_report_cap then runs the
 * local compare and the exchange in ONE kernel (publish header + flags with
 * system-scope release stores into every window, wait for all flags, merge by
 * reading the peers' packets directly; a separate exchange kernel for an empty
 * or host-resident shard) -> one host wait; no NCCL call.  A rank that never
 * arrives makes the others return ARC_E_CUDA ("peer exchange timed out")
 * after 60 s instead of hanging.
 * Setup is collective: every rank calls arc_verify_peer_export, the caller
 * all-gathers the 64-byte handles in rank order (e.g. torch.distributed), and
 * every rank calls arc_verify_peer_open.  All ranks must use the same
 * max_report_cap.  Ranks on the same GPU (different processes) work too.
 * ------------------------------------------------------------------------ */

/* Allocate this rank's window for reports of up to max_report_cap entries
 * (2 * (32 + 24 * cap) bytes + 4 KiB of flags, zeroed) and write its 64-byte
 * cudaIpcMemHandle_t to `handle`.  Re-exporting replaces the window (peers must
 * re-open).  Errors: ARC_E_NOINIT, ARC_E_INVAL (NULL handle, cap > 2^36),
 * ARC_E_NOMEM, ARC_E_CUDA. */
int arc_verify_peer_export(uint64_t max_report_cap, void *handle);

/* Map the peers' windows: `handles` = nranks x 64 bytes in rank order (the
 * own entry is ignored).  Enables the peer path.  Errors: ARC_E_NOINIT,
 * ARC_E_INVAL (no export yet, NULL handles), ARC_E_UNSUPPORTED (a handle cannot
 * be mapped, e.g. no P2P between the devices; the NCCL path stays in use). */
int arc_verify_peer_open(const void *handles);

/* Bytes this rank's exchanges have read from OTHER ranks' windows since the
 * last reset: bytes[0] = report entries pulled from the contributing ranks'
 * packets, bytes[1] = entries read from a forwarding neighbour (ring mode,
 * p >= 3 and a global report of >= 2^17 entries travels
 * owner -> owner+1 -> ... in 384 KB chunks, so no window is read more than
 * once per call).  Measured by the exchange kernels (one atomic per warp).
 * reset != 0 clears the counters.  Synchronises the library's stream.
 * Errors: ARC_E_NOINIT, ARC_E_INVAL (bytes NULL), ARC_E_CUDA. */
int arc_verify_peer_stats(uint64_t *bytes, int reset);

#ifdef __cplusplus
}
#endif
#endif /* ARC_VERIFY_H */
