"""Diagnostic: fixed vs per-byte cost of one compare call over array sizes.

For fp64 C4-generator arrays of 2^22 .. 2^29 elements (the p = 8 .. 1 shard sizes
of C4 are 2^26 .. 2^29) prints, per size: the read probe (same bulk-copy
pipeline, predicate off), the kernel window (K1 + K2 CUDA events, library
stream), the per-call device time of back-to-back prepared calls (what
bench.py's `value` measures), and the host wall time per call.  A linear fit
t = a + b * bytes over the sizes separates fixed cost (a) from streaming (b).
  python tools/size_sweep.py [f64|f32]
"""
import os
import sys
import time

sys.path.insert(0, os.getcwd())
import numpy as np
import torch

import paper_conf_ipps_leelv14_b200 as av
import synth
from synth.configs import Region

DT = sys.argv[1] if len(sys.argv) > 1 else "f64"
ES = 8 if DT == "f64" else 4
STEPS = int(os.environ.get("SWEEP_STEPS", "40"))
REP = torch.empty(24 * (1 << 20), dtype=torch.uint8, pin_memory=True).numpy().view(av.REPORT_DTYPE)

av.init(0)
stream = torch.cuda.current_stream()
rows = []
top = 29 if DT == "f64" else 30
for lg in range(22, top + 1):
    n = 1 << lg
    if DT == "f64":
        reg = synth.C4(n)
    else:
        reg = Region("F", "f32", n, 77, 1e-6, 1e-5, 1 << 20, "f32", n_inject=512)
    o, r = reg.slice(device="cuda")
    torch.cuda.synchronize()
    nb = n * ES
    probe = av.arc_verify_probe_read(o.data_ptr(), r.data_ptr(), nb, 20)
    res = {}
    for mr in (1 << 20, 0):
        step = av.prepare(o, r, reg.abs_tol, reg.rel_tol, mr, report=REP)
        for _ in range(5):
            step()
        torch.cuda.synchronize()
        av.arc_verify_set_timing(True)
        av.arc_verify_kernel_stats(reset=True)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        w0 = time.perf_counter()
        e0.record(stream)
        for _ in range(STEPS):
            step()
        e1.record(stream)
        torch.cuda.synchronize()
        wall = (time.perf_counter() - w0) / STEPS * 1e6
        k, kms = av.arc_verify_kernel_stats(reset=True)
        av.arc_verify_set_timing(False)
        res[mr] = (1e3 * kms / k, 1e3 * e0.elapsed_time(e1) / STEPS, wall)
    probe_us = 2 * nb / probe / 1e3
    k_us, call_us, wall_us = res[1 << 20]
    rows.append((2 * nb, probe_us, k_us, call_us, res[0][0]))
    print(f"{DT} n=2^{lg:<2d} read {2*nb/2**20:8.0f} MiB | probe {probe_us:8.1f} us ({probe:6.0f} GB/s) | "
          f"kernel {k_us:8.1f} us | per call {call_us:8.1f} us ({2*nb/call_us/1e3:6.0f} GB/s) wall {wall_us:8.1f} | "
          f"count-only kernel {res[0][0]:8.1f} us", flush=True)
    del o, r
    torch.cuda.empty_cache()
a = np.array(rows)
for col, name in ((1, "probe"), (2, "kernel"), (3, "per call"), (4, "count-only")):
    b, c = np.polyfit(a[:, 0], a[:, col], 1)
    print(f"fit {name:10s}: fixed {c:7.1f} us + {1e-3 / b if b else 0:7.0f} GB/s streaming "
          f"(1 / slope)", flush=True)
av.finalize()
