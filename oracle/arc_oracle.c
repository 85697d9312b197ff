/*
 * arc_oracle.c -- CPU ORACLE FOR THE KERNEL-VERIFICATION RESULT COMPARISON.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and the
 * cpu_baseline / --impl reference legs of bench.py may load or call this file.
 * The product path (paper_conf_ipps_leelv14_b200/) never links, imports or
 * executes it, and this file shares no code, header, table or constant with
 * the CUDA path.
 *
 * What it computes (PAPER.md = /root/reference/PAPER.md, cited as P:<line>):
 *   P:159  (sec. III-A) -- compare the translated GPU kernel's outputs with the
 *          sequential CPU program's outputs "at the granularity of a GPU kernel".
 *   P:171-173 (sec. III-A, Listing 2 line 11) -- "all data modified by the kernel
 *          are copied back ... result comparison codes will be added".
 *   P:199  (sec. III-A) -- "If the output difference is bigger than the allowed
 *          error margin, then an error will be reported to the user" ... "allows
 *          users to configure the error margin".
 *   P:161  -- the margin exists because CPU and GPU "use different numbers of
 *          bits" and a "non-deterministic computation order".
 * The paper gives no formula; the formula and the NaN/Inf/zero rules are the
 * readings listed in DESIGN.md sec. 3, written out here as
 * a plain, sequential, per-element definition evaluated in ascending index
 * order:
 *
 *   float dtypes (x = (double)out[i], y = (double)ref[i]; promotion is exact):
 *     rule 1  x == y                  -> match, d = 0, r = 0
 *     rule 2  isnan(x) && isnan(y)    -> match, d, r undefined (excluded)
 *     rule 3  isnan(x) || isnan(y)    -> mismatch, d, r undefined (excluded)
 *     rule 4  isinf(y)                -> mismatch, d = +Inf, r = +Inf
 *     rule 5  d = |x - y|; t = abs_tol + (rel_tol * |y|) (two RN ops, no FMA);
 *             match iff d <= t; r = (d == +Inf) ? +Inf : d / |y|
 *   integer dtypes: match iff out[i] == ref[i]; d = |out[i] - ref[i]| exactly;
 *             r undefined; tolerances ignored.
 *
 *   n_mismatch  = number of mismatches
 *   max_abs_err = max of the defined d (0 if none); integer d converted RN
 *   max_rel_err = max of the defined r (0 if none; 0 for integer dtypes)
 *   report      = the first max_report mismatching i in ascending order, each
 *                 as (i, raw bits of out[i], raw bits of ref[i]) zero-extended.
 *
 * Build: gcc -O2 -std=c99 -ffp-contract=off -fno-fast-math -shared -fPIC
 * (no -ffast-math: it would link crtfastmath and set FTZ/DAZ; no FMA
 * contraction: the tolerance is two separately rounded operations).
 *
 * Pins (tests/test_oracle.py): numpy.isclose(..., equal_nan=True) on a brute
 * force cross product of special values, hand-worked golden values in
 * tests/golden/, closed forms of the injected-mismatch generators, invariants.
 */
#include <stdint.h>
#include <string.h>
#include <math.h>
#include <stddef.h>

/* Oracle-private dtype codes (the binding in oracle/__init__.py maps names). */
enum { ORC_F32 = 0, ORC_F64 = 1, ORC_I32 = 2, ORC_I64 = 3, ORC_U8 = 4 };

typedef struct {
    uint64_t index;
    uint64_t out_bits;
    uint64_t ref_bits;
} oracle_mismatch_t;

typedef struct {
    uint64_t n;
    uint64_t n_mismatch;
    double   max_abs_err;
    double   max_rel_err;
    uint64_t n_reported;
} oracle_result_t;

/* Raw bits of element i, zero-extended to 64 bits. */
static uint64_t raw_bits(const void *a, int dtype, uint64_t i)
{
    uint64_t b = 0;
    if (dtype == ORC_F32 || dtype == ORC_I32) {
        uint32_t v;
        memcpy(&v, (const char *)a + 4 * i, 4);
        b = v;
    } else if (dtype == ORC_F64 || dtype == ORC_I64) {
        memcpy(&b, (const char *)a + 8 * i, 8);
    } else {
        b = ((const uint8_t *)a)[i];
    }
    return b;
}

static double load_float(const void *a, int dtype, uint64_t i)
{
    if (dtype == ORC_F32) {
        float v;
        memcpy(&v, (const char *)a + 4 * i, 4);
        return (double)v; /* exact widening */
    } else {
        double v;
        memcpy(&v, (const char *)a + 8 * i, 8);
        return v;
    }
}

/*
 * Per-element float rule (rules 1-5 above).  Returns 1 on mismatch.
 * *has_d / *has_r say whether d / r are defined for this element.
 */
static int float_element(double x, double y, double abs_tol, double rel_tol,
                         int *has_d, double *d_out, int *has_r, double *r_out)
{
    double d, t, ay;
    /* rule 1 */
    if (x == y) {
        *has_d = 1; *d_out = 0.0;
        *has_r = 1; *r_out = 0.0;
        return 0;
    }
    /* rule 2 */
    if (isnan(x) && isnan(y)) {
        *has_d = 0; *has_r = 0;
        return 0;
    }
    /* rule 3 */
    if (isnan(x) || isnan(y)) {
        *has_d = 0; *has_r = 0;
        return 1;
    }
    /* rule 4 */
    if (isinf(y)) {
        *has_d = 1; *d_out = INFINITY;
        *has_r = 1; *r_out = INFINITY;
        return 1;
    }
    /* rule 5 */
    d = fabs(x - y);
    ay = fabs(y);
    {
        volatile double prod = rel_tol * ay; /* separately rounded product */
        t = abs_tol + prod;                   /* separately rounded sum     */
    }
    *has_d = 1; *d_out = d;
    *has_r = 1;
    if (isinf(d))
        *r_out = INFINITY;
    else
        *r_out = d / ay; /* ay == 0 with d > 0 gives +Inf */
    return (d <= t) ? 0 : 1;
}

/* Integer |a - b| computed exactly as an unsigned magnitude. */
static uint64_t int_absdiff(const void *o, const void *r, int dtype, uint64_t i)
{
    if (dtype == ORC_I32) {
        int32_t a, b;
        memcpy(&a, (const char *)o + 4 * i, 4);
        memcpy(&b, (const char *)r + 4 * i, 4);
        int64_t diff = (int64_t)a - (int64_t)b;
        return (uint64_t)(diff < 0 ? -diff : diff);
    } else if (dtype == ORC_I64) {
        int64_t a, b;
        memcpy(&a, (const char *)o + 8 * i, 8);
        memcpy(&b, (const char *)r + 8 * i, 8);
        return a >= b ? (uint64_t)a - (uint64_t)b : (uint64_t)b - (uint64_t)a;
    } else {
        uint8_t a = ((const uint8_t *)o)[i], b = ((const uint8_t *)r)[i];
        return a >= b ? (uint64_t)(a - b) : (uint64_t)(b - a);
    }
}

/*
 * oracle_compare: the whole definition, sequential, ascending i.
 * Returns 0 on success, -1 on invalid arguments (unknown dtype, tolerances
 * NaN / negative / infinite, NULL arrays with n > 0, NULL result, NULL report
 * with max_report > 0).
 */
int oracle_compare(const void *out, const void *ref, uint64_t n, int dtype,
                   double abs_tol, double rel_tol, uint64_t max_report,
                   oracle_mismatch_t *report, oracle_result_t *res)
{
    uint64_t i;
    int is_float;
    double max_abs = 0.0, max_rel = 0.0;

    if (res == NULL) return -1;
    if (dtype < ORC_F32 || dtype > ORC_U8) return -1;
    if (!(abs_tol >= 0.0) || !(rel_tol >= 0.0) || isinf(abs_tol) || isinf(rel_tol)) return -1;
    if (n > 0 && (out == NULL || ref == NULL)) return -1;
    if (max_report > 0 && report == NULL) return -1;

    is_float = (dtype == ORC_F32 || dtype == ORC_F64);
    res->n = n;
    res->n_mismatch = 0;
    res->n_reported = 0;

    for (i = 0; i < n; ++i) {
        int mismatch;
        if (is_float) {
            int has_d, has_r;
            double d = 0.0, r = 0.0;
            double x = load_float(out, dtype, i);
            double y = load_float(ref, dtype, i);
            mismatch = float_element(x, y, abs_tol, rel_tol, &has_d, &d, &has_r, &r);
            if (has_d && d > max_abs) max_abs = d;
            if (has_r && r > max_rel) max_rel = r;
        } else {
            uint64_t m = int_absdiff(out, ref, dtype, i);
            double d = (double)m; /* RN conversion */
            mismatch = (m != 0);
            if (d > max_abs) max_abs = d;
        }
        if (mismatch) {
            if (res->n_mismatch < max_report) {
                report[res->n_mismatch].index = i;
                report[res->n_mismatch].out_bits = raw_bits(out, dtype, i);
                report[res->n_mismatch].ref_bits = raw_bits(ref, dtype, i);
            }
            res->n_mismatch += 1;
        }
    }
    res->max_abs_err = max_abs;
    res->max_rel_err = max_rel;
    res->n_reported = res->n_mismatch < max_report ? res->n_mismatch : max_report;
    return 0;
}

/*
 * oracle_compare_ex -- the same definition with the two optional checks of
 * sec. III-A / III-C (NEXT row N2; readings R10, R11 in DESIGN.md sec. 3):
 *   check_flags & 1 (minValueToCheck: "result is compared only if its value
 *       is bigger than a specified threshold"): element i is not compared when
 *       |ref[i]| <= min_value -- it is a match and its d, r are excluded.  (A NaN
 *       ref is compared: NaN <= t is false.)
 *   check_flags & 2 (value bounds: "if they fall within the user-specified
 *       bound, the tools will ignore the difference"): a mismatch with
 *       lo <= out[i] <= hi is ignored -- it is a match and its d, r are excluded.
 * Integer values enter both checks as (double) value, rounded to nearest.
 */
int oracle_compare_ex(const void *out, const void *ref, uint64_t n, int dtype,
                      double abs_tol, double rel_tol, uint64_t max_report,
                      int check_flags, double min_value, double lo, double hi,
                      oracle_mismatch_t *report, oracle_result_t *res)
{
    uint64_t i;
    int is_float;
    double max_abs = 0.0, max_rel = 0.0;

    if (res == NULL) return -1;
    if (dtype < ORC_F32 || dtype > ORC_U8) return -1;
    if (!(abs_tol >= 0.0) || !(rel_tol >= 0.0) || isinf(abs_tol) || isinf(rel_tol)) return -1;
    if (n > 0 && (out == NULL || ref == NULL)) return -1;
    if (max_report > 0 && report == NULL) return -1;
    if ((check_flags & 1) && isnan(min_value)) return -1;
    if ((check_flags & 2) && (isnan(lo) || isnan(hi))) return -1;

    is_float = (dtype == ORC_F32 || dtype == ORC_F64);
    res->n = n;
    res->n_mismatch = 0;
    res->n_reported = 0;

    for (i = 0; i < n; ++i) {
        int mismatch, has_d = 0, has_r = 0;
        double d = 0.0, r = 0.0, xv, yv;
        if (is_float) {
            xv = load_float(out, dtype, i);
            yv = load_float(ref, dtype, i);
        } else if (dtype == ORC_I32) {
            int32_t a, b;
            memcpy(&a, (const char *)out + 4 * i, 4);
            memcpy(&b, (const char *)ref + 4 * i, 4);
            xv = (double)a; yv = (double)b;
        } else if (dtype == ORC_I64) {
            int64_t a, b;
            memcpy(&a, (const char *)out + 8 * i, 8);
            memcpy(&b, (const char *)ref + 8 * i, 8);
            xv = (double)a; yv = (double)b;
        } else {
            xv = (double)((const uint8_t *)out)[i];
            yv = (double)((const uint8_t *)ref)[i];
        }
        /* check 1: not compared */
        if ((check_flags & 1) && fabs(yv) <= min_value)
            continue;
        if (is_float) {
            mismatch = float_element(xv, yv, abs_tol, rel_tol, &has_d, &d, &has_r, &r);
        } else {
            uint64_t m = int_absdiff(out, ref, dtype, i);
            d = (double)m;
            has_d = 1;
            mismatch = (m != 0);
        }
        /* check 2: an ignored difference */
        if (mismatch && (check_flags & 2) && lo <= xv && xv <= hi)
            continue;
        if (has_d && d > max_abs) max_abs = d;
        if (has_r && r > max_rel) max_rel = r;
        if (mismatch) {
            if (res->n_mismatch < max_report) {
                report[res->n_mismatch].index = i;
                report[res->n_mismatch].out_bits = raw_bits(out, dtype, i);
                report[res->n_mismatch].ref_bits = raw_bits(ref, dtype, i);
            }
            res->n_mismatch += 1;
        }
    }
    res->max_abs_err = max_abs;
    res->max_rel_err = max_rel;
    res->n_reported = res->n_mismatch < max_report ? res->n_mismatch : max_report;
    return 0;
}

/*
 * oracle_checksum -- the debug-assertion checksum (sec. III-C: "The users
 * can implement the API by performing customized bug detection (e.g.,
 * establishing checksums and verifying them)"; NEXT row N4), plain definition:
 *   words w_i = little-endian 64-bit word of bytes [8i, 8i+8), the last one
 *               zero-padded, i = 0 .. ceil(bytes/8) - 1;
 *   h_i = F(w_i + i * 0x9E3779B97F4A7C15 mod 2^64), F = the splitmix64 finalizer
 *         z ^= z >> 30; z *= 0xBF58476D1CE4E5B9; z ^= z >> 27;
 *         z *= 0x94D049BB133111EB; z ^= z >> 31;
 *   out[0] = sum of h_i mod 2^64, out[1] = xor of h_i.
 * Order-independent to reduce (any summation order gives the same value) and
 * position-dependent (moving a word changes h).
 */
static uint64_t orc_fmix(uint64_t z)
{
    z ^= z >> 30;
    z *= 0xBF58476D1CE4E5B9ull;
    z ^= z >> 27;
    z *= 0x94D049BB133111EBull;
    z ^= z >> 31;
    return z;
}

int oracle_checksum(const void *data, uint64_t bytes, uint64_t *out)
{
    uint64_t i, nw = (bytes + 7) / 8, s = 0, x = 0;
    if (out == NULL || (bytes > 0 && data == NULL)) return -1;
    for (i = 0; i < nw; ++i) {
        uint64_t w = 0, k, take = (bytes - 8 * i) < 8 ? (bytes - 8 * i) : 8;
        for (k = 0; k < take; ++k)
            w |= (uint64_t)((const uint8_t *)data)[8 * i + k] << (8 * k);
        {
            uint64_t h = orc_fmix(w + i * 0x9E3779B97F4A7C15ull);
            s += h;
            x ^= h;
        }
    }
    out[0] = s;
    out[1] = x;
    return 0;
}

/* Size check for the ctypes binding. */
size_t oracle_sizeof_result(void) { return sizeof(oracle_result_t); }
size_t oracle_sizeof_mismatch(void) { return sizeof(oracle_mismatch_t); }
