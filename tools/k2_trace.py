"""Diagnostic: per-CTA phase timeline of one compare call (K1 + K2), from a
library built with -DARCV_TRACE=1:
  python paper_conf_ipps_leelv14_b200/_build.py --variant scratch/v_trace.so -DARCV_TRACE=1
  python tools/k2_trace.py scratch/v_trace.so [log2 n]
Times in us relative to the first K1 CTA's start; min / median / max over CTAs."""
import ctypes
import os
import sys

sys.path.insert(0, os.getcwd())
import numpy as np
import torch

import paper_conf_ipps_leelv14_b200 as av
import synth

lib = ctypes.CDLL(os.path.abspath(sys.argv[1]))
lg = int(sys.argv[2]) if len(sys.argv) > 2 else 26
torch.cuda.set_device(0)
stream = torch.cuda.current_stream().cuda_stream or av.CUDA_STREAM_LEGACY
opts = av.arc_verify_opts_t(0, stream, 0, 1, None)
assert lib.arc_verify_init(ctypes.byref(opts)) == 0
REP = torch.empty(24 * (1 << 20), dtype=torch.uint8, pin_memory=True).numpy().view(av.REPORT_DTYPE)
P, U64, I, D = ctypes.c_void_p, ctypes.c_uint64, ctypes.c_int, ctypes.c_double
lib.arc_verify_compare.argtypes = [P, P, U64, I, D, D, U64, ctypes.POINTER(av.arc_verify_result_t)]
K1 = ["start", "loop end", "flush end", "exit", "first stage landed", "first tile evaluated"]
K2 = ["entry / barrier arrive", "after wait", "tile 0 emitted", "prefixes reduced", "tile 0 landed",
      "tile 0 masked", "pool loop end", "exit", "last rep start (TAIL_REPS)", "pool loaded", "tile 1 emitted",
      "after last_cta (fence+atomic+bar)"]


def run(name, o, r, at, rt, mr):
    res = av.arc_verify_result_t()
    res.report = REP.ctypes.data
    buf = np.zeros((3, 1024, 32), dtype=np.uint64)
    for it in range(5):
        if it == 4:  # clear the stamps: the traced call is the last one
            lib.arc_verify_debug_trace(buf.ctypes.data_as(ctypes.POINTER(ctypes.c_ulonglong)))
        assert lib.arc_verify_compare(o.data_ptr(), r.data_ptr(), o.numel(), av.dtype_code(o), at, rt, mr,
                                      ctypes.byref(res)) == 0
    buf = np.zeros((3, 1024, 32), dtype=np.uint64)
    assert lib.arc_verify_debug_trace(buf.ctypes.data_as(ctypes.POINTER(ctypes.c_ulonglong))) == 0
    t = buf.astype(np.float64)
    k1 = t[0][t[0][:, 0] > 0]
    k2 = t[1][t[1][:, 0] > 0]
    t0 = k1[:, 0].min()
    print(f"== {name}: {len(k1)} K1 CTAs, {len(k2)} K2 CTAs, mismatches {res.n_mismatch}")
    for arr, names, kn in ((k1, K1, "K1"), (k2, K2, "K2")):
        for i, nm in enumerate(names):
            col = arr[:, i]
            col = col[col > 0]
            if len(col):
                d = (col - t0) / 1e3
                print(f"  {kn} {nm:18s} min {d.min():8.2f}  med {np.median(d):8.2f}  max {d.max():8.2f}  (n={len(col)})")


def run_probe(name, o, r):
    """The read probe (same K1 pipeline, predicate off) traced like a compare."""
    buf = np.zeros((3, 1024, 32), dtype=np.uint64)
    lib.arc_verify_probe_read.argtypes = [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_uint64, ctypes.c_int,
                                          ctypes.POINTER(ctypes.c_double)]
    g = ctypes.c_double()
    lib.arc_verify_probe_read(o.data_ptr(), r.data_ptr(), o.numel() * o.element_size(), 3, ctypes.byref(g))
    lib.arc_verify_debug_trace(buf.ctypes.data_as(ctypes.POINTER(ctypes.c_ulonglong)))  # clear
    assert lib.arc_verify_probe_read(o.data_ptr(), r.data_ptr(), o.numel() * o.element_size(), 1,
                                     ctypes.byref(g)) == 0
    assert lib.arc_verify_debug_trace(buf.ctypes.data_as(ctypes.POINTER(ctypes.c_ulonglong))) == 0
    t = buf.astype(np.float64)
    k1 = t[0][t[0][:, 0] > 0]
    t0 = k1[:, 0].min()
    print(f"== {name}: {len(k1)} K1 CTAs (probe: {g.value:.0f} GB/s event-timed)")
    for i, nm in enumerate(K1):
        col = k1[:, i]
        col = col[col > 0]
        if len(col):
            d = (col - t0) / 1e3
            print(f"  K1 {nm:18s} min {d.min():8.2f}  med {np.median(d):8.2f}  max {d.max():8.2f}  (n={len(col)})")


if os.environ.get("TRACE_C5"):
    c5 = synth.C5(1 << int(os.environ.get("TRACE_C5_LOG2", "30")))
    o, r = c5.slice(device="cuda")
    rep = torch.empty(24 * c5.max_report, dtype=torch.uint8, device="cuda")
    run(f"C5 int32 2^{int(os.environ.get('TRACE_C5_LOG2', '30'))}, 50% mismatches, max_report 2^20 (pinned report)",
        o, r, 0.0, 0.0, c5.max_report)
    run("C5, count only", o, r, 0.0, 0.0, 0)
elif os.environ.get("TRACE_C2A"):
    c2 = synth.C2("A")
    o, r = c2.slice(device="cuda")
    run_probe("read probe over the C2A arrays", o, r)
    run("C2A fp32 8192^2, max_report 2^20", o, r, c2.abs_tol, c2.rel_tol, c2.max_report)
    run("C2A fp32 8192^2, count only", o, r, c2.abs_tol, c2.rel_tol, 0)
    run("C2A bytes as u8 (no float filter), count only", o.view(torch.uint8), r.view(torch.uint8), 0, 0, 0)
    c2b = synth.C2("B")
    o, r = c2b.slice(device="cuda")
    run("C2B fp32 8192^2 (2 dense tiles), pinned report 2^20", o, r, c2b.abs_tol, c2b.rel_tol, c2b.max_report)
    c1 = synth.C1()
    o, r = c1.slice(device="cuda")
    run("C1 fp32 2^20, pinned report 2^20", o, r, c1.abs_tol, c1.rel_tol, c1.max_report)
else:
    c = synth.C4(1 << lg)
    o, r = c.slice(device="cuda")
    run(f"C4 fp64 2^{lg}, max_report 2^20", o, r, c.abs_tol, c.rel_tol, c.max_report)
    run(f"C4 fp64 2^{lg}, count only", o, r, c.abs_tol, c.rel_tol, 0)
