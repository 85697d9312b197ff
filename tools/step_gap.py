"""Diagnostic: where the time between two back-to-back C4 calls goes.
Per step (CUDA events around K back-to-back calls) vs the kernel alone (library
events around each launch), for the Python prepared call and for raw ctypes, plus
host wall time per call.
  python tools/step_gap.py"""
import ctypes
import os
import sys
import time

sys.path.insert(0, os.getcwd())
import torch

import paper_conf_ipps_leelv14_b200 as av
import synth

K = int(os.environ.get("SG_STEPS", "200"))
av.init(0)
c4 = synth.C4()
o, r = c4.slice(device="cuda")
rep = torch.empty(24 * c4.max_report, dtype=torch.uint8, pin_memory=True).numpy().view(av.REPORT_DTYPE)
step = av.prepare(o, r, c4.abs_tol, c4.rel_tol, c4.max_report, report=rep)
res = av.arc_verify_result_t()
res.report = rep.ctypes.data
f, br, po, pr, n = av._lib.arc_verify_compare, ctypes.byref(res), o.data_ptr(), r.data_ptr(), o.numel()
raw = lambda: f(po, pr, n, 1, c4.abs_tol, c4.rel_tol, c4.max_report, br)
stream = torch.cuda.current_stream()
for _ in range(5):
    step()
torch.cuda.synchronize()


def per_step(fn):
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    w0 = time.perf_counter()
    e0.record(stream)
    for _ in range(K):
        fn()
    e1.record(stream)
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / K * 1e3, (time.perf_counter() - w0) / K * 1e6


def kernel(fn):
    av.arc_verify_set_timing(True)
    av.arc_verify_kernel_stats(reset=True)
    for _ in range(K):
        fn()
    torch.cuda.synchronize()
    nl, ms = av.arc_verify_kernel_stats(reset=True)
    av.arc_verify_set_timing(False)
    return 1e3 * ms / max(nl, 1)


for rd in range(3):
    for name, fn in (("prepared", step), ("raw ctypes", raw)):
        ps, wall = per_step(fn)
        kr = kernel(fn)
        print(f"{name:10s}: per step {ps:7.1f} us (wall {wall:7.1f}) | kernel {kr:7.1f} us | gap {ps - kr:5.1f} us",
              flush=True)
