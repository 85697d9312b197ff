// arcv_report.cu -- NEXT row N3: region selection and report printing (host).
//
// Sec. III-A: "a user can specify which specific kernels to verify by
// adding directives or using environment variables (e.g.,
// "verificationOptions=complement=0,kernels=main_kernel0" informs the compiler
// to verify a specific kernel, main_kernel0.)"; "an error will be
// reported to the user".  Reading (R20): options are comma-separated
// key=value pairs; `kernels` lists region names separated by ':' (further
// comma-separated tokens without '=' are also names); complement=0 (default)
// verifies only the listed regions, complement=1 verifies all but them; no
// `kernels` key selects every region.  options == NULL reads the environment
// variable `verificationOptions` (then `ARC_VERIFICATION_OPTIONS`); unset means
// every region is verified.
#include <cuda_runtime.h>

#include <cinttypes>
#include <cmath>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <string>
#include <vector>

#include "arc_verify.h"
#include "arcv_internal.h"

namespace arcv {

struct Selection {
    bool complement = false;
    bool has_list = false;
    std::vector<std::string> names;
};

static std::string trim(const std::string &s) {
    size_t a = s.find_first_not_of(" \t\n\r"), b = s.find_last_not_of(" \t\n\r");
    return a == std::string::npos ? std::string() : s.substr(a, b - a + 1);
}

static int parse_options(const char *opts, Selection &sel) {
    std::string s = opts ? opts : "";
    const std::string prefix = "verificationOptions=";
    if (s.compare(0, prefix.size(), prefix) == 0) s = s.substr(prefix.size());
    size_t pos = 0;
    bool in_kernels = false;
    while (pos <= s.size()) {
        size_t comma = s.find(',', pos);
        if (comma == std::string::npos) comma = s.size();
        const std::string tok = trim(s.substr(pos, comma - pos));
        pos = comma + 1;
        if (tok.empty()) continue;
        const size_t eq = tok.find('=');
        if (eq == std::string::npos) {
            if (!in_kernels) {
                set_error("verificationOptions: token '%s' is not key=value", tok.c_str());
                return ARC_E_INVAL;
            }
            sel.names.push_back(tok);
            continue;
        }
        const std::string key = trim(tok.substr(0, eq)), val = trim(tok.substr(eq + 1));
        in_kernels = false;
        if (key == "complement") {
            if (val != "0" && val != "1") {
                set_error("verificationOptions: complement must be 0 or 1, got '%s'", val.c_str());
                return ARC_E_INVAL;
            }
            sel.complement = val == "1";
        } else if (key == "kernels") {
            sel.has_list = true;
            in_kernels = true;
            size_t p = 0;
            while (p <= val.size()) {
                size_t c = val.find(':', p);
                if (c == std::string::npos) c = val.size();
                const std::string nm = trim(val.substr(p, c - p));
                if (!nm.empty()) sel.names.push_back(nm);
                p = c + 1;
            }
        }  // other OpenARC options are not ours: ignored
    }
    return ARC_OK;
}

static const char *env_options() {
    const char *e = getenv("verificationOptions");
    if (!e || !*e) e = getenv("ARC_VERIFICATION_OPTIONS");
    return (e && *e) ? e : nullptr;
}

static bool is_selected(const Selection &sel, const char *name) {
    if (!sel.has_list) return true;  // no list: every region
    bool listed = false;
    if (name)
        for (const auto &n : sel.names) listed |= (n == name);
    return sel.complement ? !listed : listed;
}

static void fmt_value(char *b, size_t cap, uint64_t bits, int dtype) {
    switch (dtype) {
        case ARC_F32: {
            float f;
            uint32_t u = (uint32_t)bits;
            memcpy(&f, &u, 4);
            snprintf(b, cap, "%.9g (0x%08" PRIx32 ")", (double)f, u);
            break;
        }
        case ARC_F64: {
            double d;
            memcpy(&d, &bits, 8);
            snprintf(b, cap, "%.17g (0x%016" PRIx64 ")", d, bits);
            break;
        }
        case ARC_I32: snprintf(b, cap, "%" PRId32, (int32_t)(uint32_t)bits); break;
        case ARC_I64: snprintf(b, cap, "%" PRId64, (int64_t)bits); break;
        default: snprintf(b, cap, "%" PRIu64, bits); break;
    }
}

}  // namespace arcv

using namespace arcv;

extern "C" {

int arc_verify_selected(const char *options, const char *name) {
    if (!options) options = env_options();
    if (!options) return 1;
    Selection sel;
    int st = parse_options(options, sel);
    if (st) return st;
    return is_selected(sel, name) ? 1 : 0;
}

int arc_verify_batch_selected(const arc_verify_region_t *regions, size_t n_regions, const char *options,
                              arc_verify_result_t *results, uint8_t *selected) {
    if (!g_ctx) return ARC_E_NOINIT;
    if (n_regions == 0) return ARC_OK;
    if (!regions || !results) {
        set_error("regions/results is NULL");
        return ARC_E_INVAL;
    }
    if (!options) options = env_options();
    Selection sel;
    if (options) {
        int st = parse_options(options, sel);
        if (st) return st;
    }
    std::vector<arc_verify_region_t> sub;
    std::vector<arc_verify_result_t> subres;
    std::vector<size_t> where;
    for (size_t k = 0; k < n_regions; ++k) {
        const bool on = !options || is_selected(sel, regions[k].name);
        if (selected) selected[k] = on ? 1 : 0;
        if (!on) {
            arc_mismatch_t *rep = results[k].report;
            memset(&results[k], 0, sizeof(results[k]));
            results[k].report = rep;
            continue;
        }
        sub.push_back(regions[k]);
        subres.push_back(results[k]);
        where.push_back(k);
    }
    if (sub.empty()) return ARC_OK;
    int st = arc_verify_batch(sub.data(), sub.size(), subres.data());
    if (st) return st;
    for (size_t j = 0; j < where.size(); ++j) results[where[j]] = subres[j];
    return ARC_OK;
}

int arc_verify_format_result(const char *name, arc_dtype_t dtype, double abs_tol, double rel_tol,
                             const arc_verify_result_t *result, uint64_t max_entries, char *buf, size_t cap) {
    if (!result || !buf || cap == 0 || dtype < ARC_F32 || dtype > ARC_U8) {
        set_error("format_result: bad arguments");
        return ARC_E_INVAL;
    }
    if (max_entries > 0 && result->n_reported > 0 && !result->report) {
        set_error("format_result: report is NULL");
        return ARC_E_INVAL;
    }
    std::string s;
    char line[512];
    const bool is_float = dtype == ARC_F32 || dtype == ARC_F64;
    snprintf(line, sizeof(line), "[arc_verify] %s: %s -- %" PRIu64 " of %" PRIu64 " elements differ", name ? name : "(region)",
             result->n_mismatch ? "FAILED" : "passed", result->n_mismatch, result->n);
    s += line;
    if (is_float)
        snprintf(line, sizeof(line), " (abs_tol=%g, rel_tol=%g); max_abs_err=%.17g max_rel_err=%.17g", abs_tol,
                 rel_tol, result->max_abs_err, result->max_rel_err);
    else
        snprintf(line, sizeof(line), " (exact); max_abs_err=%.17g", result->max_abs_err);
    s += line;
    const uint64_t show = result->n_reported < max_entries ? result->n_reported : max_entries;
    if (show) {
        snprintf(line, sizeof(line), "; first %" PRIu64 " of %" PRIu64 " reported:", show, result->n_reported);
        s += line;
    }
    s += "\n";
    // entries: the report may be device memory -- copy what we print
    std::vector<arc_mismatch_t> ent(show);
    if (show) {
        cudaPointerAttributes a;
        bool dev = false;
        if (cudaPointerGetAttributes(&a, result->report) == cudaSuccess)
            dev = a.type == cudaMemoryTypeDevice || a.type == cudaMemoryTypeManaged;
        else
            cudaGetLastError();
        if (dev) {
            cudaError_t e = cudaMemcpy(ent.data(), result->report, show * sizeof(arc_mismatch_t),
                                       cudaMemcpyDeviceToHost);
            if (e != cudaSuccess) return cuda_fail(e, "cudaMemcpy(report entries)");
        } else {
            memcpy(ent.data(), result->report, show * sizeof(arc_mismatch_t));
        }
    }
    for (uint64_t i = 0; i < show; ++i) {
        char vo[96], vr[96];
        fmt_value(vo, sizeof(vo), ent[i].out_bits, dtype);
        fmt_value(vr, sizeof(vr), ent[i].ref_bits, dtype);
        snprintf(line, sizeof(line), "  [%" PRIu64 "] out=%s ref=%s\n", ent[i].index, vo, vr);
        s += line;
    }
    const size_t n = s.size() < cap - 1 ? s.size() : cap - 1;
    memcpy(buf, s.data(), n);
    buf[n] = '\0';
    return (int)std::min<size_t>(s.size(), 0x7fffffff);
}

}  // extern "C"
