// arcv_merge.h -- the cross-GPU merge plan (DESIGN.md sec. 2 step a8, reading
// R-shard): one definition shared by the host entry point, the NCCL-path merge
// kernel and the peer-memory exchange kernel.
#pragma once
#include <cstdint>

#include "arc_verify.h"

namespace arcv {

constexpr int kMaxRanks = 256;

// Shards are contiguous ascending index ranges in rank order, so the global
// report is the rank-order concatenation: rank r starts at report position
// prefix_r (mismatches of lower ranks) and contributes what still fits.
__host__ __device__ inline void merge_plan_impl(const arc_shard_header_t *h, int p, uint64_t max_report,
                                                arc_shard_plan_t *plan, arc_shard_header_t *g) {
    uint64_t off = 0, pre = 0;
    g->n = 0;
    g->n_mismatch = 0;
    g->max_abs_bits = 0;
    g->max_rel_bits = 0;
    for (int r = 0; r < p; ++r) {
        plan[r].index_offset = off;
        plan[r].prefix = pre;
        const uint64_t rem = max_report > pre ? max_report - pre : 0;
        plan[r].contrib = h[r].n_mismatch < rem ? h[r].n_mismatch : rem;
        off += h[r].n;
        pre += h[r].n_mismatch;
        g->n += h[r].n;
        g->n_mismatch += h[r].n_mismatch;
        g->max_abs_bits = h[r].max_abs_bits > g->max_abs_bits ? h[r].max_abs_bits : g->max_abs_bits;
        g->max_rel_bits = h[r].max_rel_bits > g->max_rel_bits ? h[r].max_rel_bits : g->max_rel_bits;
    }
}

}  // namespace arcv
