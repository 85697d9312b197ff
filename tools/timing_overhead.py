"""Diagnostic: what the library's per-launch timing events (arc_verify_set_timing,
two cudaEventRecord per launch, ~2.6 us of host time each on these boxes) add to a
bench step -- per-step device time of K back-to-back prepared compares (torch
events around the loop, as bench.py times `value`) with the library timing on
and off, at the p = 8 shard size and the full C4 size.
  python tools/timing_overhead.py"""
import os
import sys

sys.path.insert(0, os.getcwd())
import torch

import paper_conf_ipps_leelv14_b200 as av
import synth

av.init(0)
stream = torch.cuda.current_stream()
rep = torch.empty(24 << 20, dtype=torch.uint8, pin_memory=True).numpy().view(av.REPORT_DTYPE)
for lg in (26, 29):
    c = synth.C4(1 << lg)
    o, r = c.slice(device="cuda")
    step = av.prepare(o, r, c.abs_tol, c.rel_tol, c.max_report, report=rep)
    for _ in range(5):
        step()
    res = {}
    for rnd in range(3):
        for timing in (True, False):
            av.arc_verify_set_timing(timing)
            av.arc_verify_kernel_stats(reset=True)
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            k = 40 if lg == 26 else 10
            e0.record(stream)
            for _ in range(k):
                step()
            e1.record(stream)
            torch.cuda.synchronize()
            n, kms = av.arc_verify_kernel_stats(reset=True)
            res.setdefault(timing, []).append((1e3 * e0.elapsed_time(e1) / k, 1e3 * kms / n if n else None))
    av.arc_verify_set_timing(False)
    for timing in (True, False):
        steps = sorted(x[0] for x in res[timing])
        kern = [x[1] for x in res[timing] if x[1]]
        print(f"C4 2^{lg}: library timing {'on ' if timing else 'off'}: per step {steps[len(steps) // 2]:8.1f} us (median of 3)"
              + (f", kernel events {sorted(kern)[len(kern) // 2]:8.1f} us" if kern else ""))
    del o, r
    torch.cuda.empty_cache()
av.finalize()
