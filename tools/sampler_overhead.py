"""Diagnostic: does the NVML clock sampler thread (bench.py ClockSampler) slow the
timed bench loop?  C4 prepared calls, K steps timed with CUDA events, with no sampler
and with the sampler polling every 5 / 50 ms, interleaved.
  python tools/sampler_overhead.py"""
import os
import sys
import time

sys.path.insert(0, os.getcwd())
import torch

import bench
import paper_conf_ipps_leelv14_b200 as av
import synth

STEPS = int(os.environ.get("SO_STEPS", "200"))
av.init(0)
c4 = synth.C4()
o, r = c4.slice(device="cuda")
rep = torch.empty(24 * c4.max_report, dtype=torch.uint8, pin_memory=True).numpy().view(av.REPORT_DTYPE)
step = av.prepare(o, r, c4.abs_tol, c4.rel_tol, c4.max_report, report=rep)
stream = torch.cuda.current_stream()
for _ in range(5):
    step()
torch.cuda.synchronize()


def run(interval):
    s = None
    if interval is not None:
        s = bench.ClockSampler(0)
        s.interval = interval
        s.__enter__()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(stream)
    for _ in range(STEPS):
        step()
    e1.record(stream)
    torch.cuda.synchronize()
    if s is not None:
        s.__exit__()
    return e0.elapsed_time(e1) / STEPS * 1e3


res = {None: [], 0.005: [], 0.05: []}
for rd in range(4):
    for iv in (None, 0.005, 0.05):
        res[iv].append(run(iv))
for iv, v in res.items():
    print(f"sampler {'off' if iv is None else f'{iv * 1e3:.0f} ms'}: per step " + " ".join(f"{x:.1f}" for x in v) +
          f" us (min {min(v):.1f})", flush=True)
