"""NVLink bytes moved by the sharded exchange, per rank, for the north_star
shapes (C4: fp64 2^29, 516 sparse mismatches; C5: int32 2^30, 50 % mismatches,
max_report 2^20) at p = 2 / 4 / 8 -- pull-from-owner vs ring forwarding
(csrc/arcv_exchange.cuh).  Host only: the merge plan comes
from the library's own arc_verify_merge_plan (no GPU needed); the byte rules
are the ones the exchange kernel applies, and tests/test_peer_scale_gpu.py
checks them against the kernel's measured counters (arc_verify_peer_stats).

  python tools/exchange_bytes.py
"""
import os
import sys

sys.path.insert(0, os.getcwd())
import paper_conf_ipps_leelv14_b200 as av  # noqa: E402

ENTRY = 24
RING_MIN = 1 << 17      # kRingMin (entries)
RING_CHUNK = 1 << 14    # kRingChunk (entries)
LINK_GBS = 750.0        # assumed achievable NVLink 5 pull bandwidth per GPU and direction


def headers(cfg, p):
    n = 1 << 29 if cfg == "C4" else 1 << 30
    hs = []
    for r in range(p):
        lo, hi = r * n // p, (r + 1) * n // p
        if cfg == "C4":  # 516 planted mismatches, spread uniformly (closed form of the generator)
            mis = 516 * (hi - lo) // n + (1 if r < 516 % p else 0)
        else:            # every odd index
            mis = hi // 2 - lo // 2
        hs.append((hi - lo, mis, 0, 0))
    return hs


def bytes_moved(cfg, p, max_report=1 << 20):
    plan, g = av.arc_verify_merge_plan(headers(cfg, p), max_report)
    contrib = [c for (_off, _pre, c) in plan]
    total = sum(contrib)
    ring = p >= 3 and total >= RING_MIN
    ingress, egress = [0] * p, [0] * p
    for q, c in enumerate(contrib):
        if not c:
            continue
        if ring:  # q -> q+1 -> ... -> q-1: each hop reads the chunk once from its predecessor
            for k in range(1, p):
                dst, src = (q + k) % p, (q + k - 1) % p
                ingress[dst] += c * ENTRY
                egress[src] += c * ENTRY
        else:     # every other rank pulls q's entries from q's window
            for r in range(p):
                if r != q:
                    ingress[r] += c * ENTRY
                    egress[q] += c * ENTRY
    chunks = sum((c + RING_CHUNK - 1) // RING_CHUNK for c in contrib)
    return {"mode": "ring" if ring else "pull", "total_entries": total, "ingress": ingress, "egress": egress,
            "chunks": chunks, "bound_us": max(max(ingress), max(egress)) / (LINK_GBS * 1e3)}


def main():
    print(f"{'cfg':4s} {'p':>2s} {'mode':5s} {'entries':>9s} {'max egress/rank':>16s} {'max ingress/rank':>17s}"
          f" {'link-bound us':>13s}   (pull at the same p: max egress, us)")
    for cfg in ("C4", "C5"):
        for p in (2, 4, 8):
            d = bytes_moved(cfg, p)
            plan, _ = av.arc_verify_merge_plan(headers(cfg, p), 1 << 20)
            pull_egress = max(c * ENTRY * (p - 1) for (_o, _p, c) in plan)
            print(f"{cfg:4s} {p:2d} {d['mode']:5s} {d['total_entries']:9d} {max(d['egress']) / 2**20:13.2f} MiB"
                  f" {max(d['ingress']) / 2**20:14.2f} MiB {d['bound_us']:13.1f}   "
                  f"({pull_egress / 2**20:.2f} MiB, {pull_egress / (LINK_GBS * 1e3):.1f} us)")


if __name__ == "__main__":
    main()
