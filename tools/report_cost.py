"""Diagnostic: what the sparse report adds to a mid-size call (C4 fp64 at 2^24 /
2^26 elements, 516 planted-density mismatches): kernel time (library CUDA
events, idle stream before each call) for count-only, a device-memory report,
a pinned host report and a pageable one, against the read probe.
  python tools/report_cost.py"""
import os
import sys

sys.path.insert(0, os.getcwd())
import numpy as np
import torch

import paper_conf_ipps_leelv14_b200 as av
import synth

av.init(0)


def kt(fn, steps=30):
    for _ in range(3):
        fn()
    torch.cuda.synchronize()
    av.arc_verify_set_timing(True)
    av.arc_verify_kernel_stats(reset=True)
    for _ in range(steps):
        fn()
    torch.cuda.synchronize()
    n, ms = av.arc_verify_kernel_stats(reset=True)
    av.arc_verify_set_timing(False)
    return 1e3 * ms / n


for lg in (24, 26):
    c = synth.C4(1 << lg)
    o, r = c.slice(device="cuda")
    nb = o.numel() * 8
    pin = torch.empty(24 << 20, dtype=torch.uint8, pin_memory=True).numpy().view(av.REPORT_DTYPE)
    page = np.zeros(1 << 20, dtype=av.REPORT_DTYPE)
    dev = torch.empty(24 << 20, dtype=torch.uint8, device="cuda")
    probe = 2 * nb / av.arc_verify_probe_read(o.data_ptr(), r.data_ptr(), nb, 30) / 1e3
    rows = [("probe (isolated launches)", probe)]
    for name, mr, rep in (("count-only", 0, None), ("device report", 1 << 20, dev),
                          ("pinned report", 1 << 20, pin), ("pageable report", 1 << 20, page)):
        p = av.prepare(o, r, c.abs_tol, c.rel_tol, mr, report=rep)
        rows.append((name, kt(p)))
    g = av.compare(o, r, c.abs_tol, c.rel_tol, 1 << 20)
    print(f"C4 2^{lg} ({2 * nb / 2**20:.0f} MiB read, {g.n_mismatch} mismatches): " +
          " | ".join(f"{k} {v:7.1f} us" for k, v in rows))
av.finalize()
