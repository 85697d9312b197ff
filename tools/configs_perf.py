"""Diagnostic: per-call device time of every BASELINE config at p = 1.

C1 (fp32 2^20, specials), C2 A/B (Jacobi-2D 8192^2 fp32), C3 (twelve regions:
one arc_verify_batch vs twelve arc_verify_compare calls), C5 (int32 2^30, 50 %
mismatches, max_report 2^20; report to pinned host and to device memory).
For each: the read probe over the same bytes, the kernel window (library CUDA
events), and the per-call device time of back-to-back calls (torch events on
the library's stream).  Arrays smaller than 4x L2 get an L2 flush (a 2x L2
scratch write) between calls, outside the per-call events.
  python tools/configs_perf.py
"""
import os
import sys

sys.path.insert(0, os.getcwd())
import torch

import paper_conf_ipps_leelv14_b200 as av
import synth

STEPS = int(os.environ.get("CFG_STEPS", "20"))
L2 = torch.cuda.get_device_properties(0).L2_cache_size if torch.cuda.is_available() else 0
REP = torch.empty(24 * (1 << 20), dtype=torch.uint8, pin_memory=True).numpy().view(av.REPORT_DTYPE)
stream = None


def timed(fn, nbytes, flush):
    scratch = torch.empty(2 * L2, dtype=torch.uint8, device="cuda") if flush else None
    for _ in range(3):
        fn()
    torch.cuda.synchronize()
    av.arc_verify_set_timing(True)
    av.arc_verify_kernel_stats(reset=True)
    tot = 0.0
    for _ in range(STEPS):
        if flush:
            scratch.fill_(1)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        fn()
        e1.record(stream)
        torch.cuda.synchronize()
        tot += e0.elapsed_time(e1)
    k, kms = av.arc_verify_kernel_stats(reset=True)
    av.arc_verify_set_timing(False)
    call_us = 1e3 * tot / STEPS
    kern_us = 1e3 * kms / max(k, 1) * (k / STEPS if k else 0)  # all launches of one call
    return call_us, kern_us


def line(name, nbytes, call_us, kern_us, probe_gbs, extra=""):
    print(f"{name:34s} {nbytes / 2**20:8.1f} MiB | per call {call_us:8.1f} us ({nbytes / call_us / 1e3:6.0f} GB/s) "
          f"| kernel {kern_us:8.1f} us ({nbytes / kern_us / 1e3 if kern_us else 0:6.0f} GB/s) "
          f"| probe {probe_gbs:6.0f} GB/s {extra}", flush=True)


def main():
    global stream
    av.init(0)
    stream = torch.cuda.current_stream()
    # C1
    c1 = synth.C1()
    o, r = c1.slice(device="cuda")
    nb = 2 * o.numel() * 4
    pr = av.arc_verify_probe_read(o.data_ptr(), r.data_ptr(), nb // 2, 50)
    st = av.prepare(o, r, c1.abs_tol, c1.rel_tol, c1.max_report, report=REP)
    res = st()
    line("C1 fp32 2^20", nb, *timed(st, nb, True), pr, f"mism={res.n_mismatch}")
    del o, r
    # C2
    for var in ("A", "B"):
        c2 = synth.C2(var)
        o, r = c2.slice(device="cuda")
        nb = 2 * o.numel() * 4
        pr = av.arc_verify_probe_read(o.data_ptr(), r.data_ptr(), nb // 2, 20)
        st = av.prepare(o, r, c2.abs_tol, c2.rel_tol, c2.max_report, report=REP)
        res = st()
        line(f"C2{var} Jacobi fp32 8192^2", nb, *timed(st, nb, False), pr, f"mism={res.n_mismatch}")
        del o, r
    # C3
    regs = synth.c3_regions()
    data = [rg.slice(device="cuda") for rg in regs]
    nb = sum(2 * o.numel() * o.element_size() for o, _ in data)
    tup = [(o, r, rg.abs_tol, rg.rel_tol, rg.max_report, rg.name) for rg, (o, r) in zip(regs, data)]
    pb = av.prepare_batch(tup)
    b = pb()
    line("C3 batch (1 call, 12 regions)", nb, *timed(pb, nb, True), 0.0,
         f"mism={sum(x.n_mismatch for x in b)}")
    singles = [av.prepare(o, r, rg.abs_tol, rg.rel_tol, rg.max_report) for rg, (o, r) in zip(regs, data)]

    def run12():
        for s in singles:
            s()
    line("C3 12 single calls", nb, *timed(run12, nb, True), 0.0)
    del data, tup, singles
    # C5
    c5 = synth.C5()
    o, r = c5.slice(device="cuda")
    nb = 2 * o.numel() * 4
    pr = av.arc_verify_probe_read(o.data_ptr(), r.data_ptr(), nb // 2, 10)
    st = av.prepare(o, r, 0, 0, c5.max_report, report=REP)
    res = st()
    line("C5 int32 2^30 dense, host report", nb, *timed(st, nb, False), pr, f"mism={res.n_mismatch}")
    drep = torch.empty(24 * c5.max_report, dtype=torch.uint8, device="cuda")
    st = av.prepare(o, r, 0, 0, c5.max_report, report=drep)
    line("C5 int32 2^30 dense, device report", nb, *timed(st, nb, False), pr)
    st = av.prepare(o, r, 0, 0, 0, report=REP)
    line("C5 int32 2^30 dense, count only", nb, *timed(st, nb, False), pr)
    st = av.prepare(o, o, 0, 0, c5.max_report, report=REP)
    line("C5-size int32 clean (out==ref)", nb, *timed(st, nb, False), pr)
    av.finalize()


if __name__ == "__main__":
    main()
