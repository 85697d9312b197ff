"""Diagnostic: cost of entering a region in a batched grid, per CTA, from a
-DARCV_TRACE=1 build (row 2 of the trace: switch into segment k / its first
tile evaluated).  Prints, per segment, how many CTAs entered it and the
first-tile time (switch -> first tile evaluated: accumulator flush of the
previous region, filter seeding, the tile itself) against a steady-state tile.
  python tools/region_trace.py scratch/v_trace.so
"""
import ctypes
import os
import sys

sys.path.insert(0, os.getcwd())
import numpy as np
import torch

import paper_conf_ipps_leelv14_b200 as av
import synth
from synth.configs import Region

lib = ctypes.CDLL(os.path.abspath(sys.argv[1]))
torch.cuda.set_device(0)
stream = torch.cuda.current_stream().cuda_stream or av.CUDA_STREAM_LEGACY
assert lib.arc_verify_init(ctypes.byref(av.arc_verify_opts_t(0, stream, 0, 1, None))) == 0
lib.arc_verify_batch.argtypes = [ctypes.POINTER(av.arc_verify_region_t), ctypes.c_size_t,
                                 ctypes.POINTER(av.arc_verify_result_t)]
BUF = np.zeros((3, 1024, 32), dtype=np.uint64)


def run(name, pairs):
    R = (av.arc_verify_region_t * len(pairs))()
    res = (av.arc_verify_result_t * len(pairs))()
    for i, (o, r, at, rt) in enumerate(pairs):
        R[i].out, R[i].ref, R[i].n = o.data_ptr(), r.data_ptr(), o.numel()
        R[i].dtype, R[i].abs_tol, R[i].rel_tol, R[i].max_report = av.dtype_code(o), at, rt, 0
    for it in range(5):
        if it == 4:
            lib.arc_verify_debug_trace(BUF.ctypes.data_as(ctypes.POINTER(ctypes.c_ulonglong)))
        assert lib.arc_verify_batch(R, len(pairs), res) == 0
    BUF[:] = 0
    assert lib.arc_verify_debug_trace(BUF.ctypes.data_as(ctypes.POINTER(ctypes.c_ulonglong))) == 0
    t = BUF.astype(np.float64)
    k1 = t[0][t[0][:, 0] > 0]
    t0 = k1[:, 0].min()
    loop = (np.median(k1[:, 1]) - t0) / 1e3
    ntiles = sum((o.numel() * o.element_size() + 16383) // 16384 for o, _, _, _ in pairs)
    ctas = len(k1)
    steady = loop / (ntiles / ctas)
    print(f"== {name}: {ctas} CTAs, loop end (median) {loop:.1f} us, {ntiles} tiles -> {steady:.2f} us per tile per CTA")
    rows = t[2]
    for s in range(min(16, len(pairs))):
        a, b = rows[:, 2 * s], rows[:, 2 * s + 1]
        m = (a > 0) & (b > 0)
        if not m.any():
            continue
        d = (b[m] - a[m]) / 1e3
        print(f"  seg {s:2d} ({pairs[s][0].dtype}, {pairs[s][0].numel() * pairs[s][0].element_size() / 2**20:7.1f} MiB):"
              f" {m.sum():4d} CTAs entered at {np.median((a[m] - t0) / 1e3):7.1f} us (median); first tile"
              f" med {np.median(d):5.2f} us, p90 {np.percentile(d, 90):5.2f}, max {d.max():5.2f}")


n = 12 * (1 << 22)
for dt in ("f32", "i32"):
    at, rt = (1e-6, 1e-5) if dt == "f32" else (0, 0)
    reg = Region("F", dt, n, 91, at, rt, 0, dt, n_inject=24)
    o, r = reg.slice(device="cuda")
    m = n // 12
    run(f"twelve equal {dt} regions, count only", [(o[k * m:(k + 1) * m], r[k * m:(k + 1) * m], at, rt) for k in range(12)])
regs = synth.c3_regions()
data = [rg.slice(device="cuda") for rg in regs]
order = sorted(range(12), key=lambda k: data[k][0].numel() * data[k][0].element_size())
run("C3 (smallest first), count only", [(data[k][0], data[k][1], regs[k].abs_tol, regs[k].rel_tol) for k in order])
