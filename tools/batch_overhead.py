"""Diagnostic: per-region overhead of one batched grid -- the same bytes as one
region, as 12 equal regions, and as the C3 set (kernel window per call)."""
import os
import sys

sys.path.insert(0, os.getcwd())
import torch

import paper_conf_ipps_leelv14_b200 as av
import synth
from synth.configs import Region

STEPS = 20


def kern(fn):
    for _ in range(3):
        fn()
    torch.cuda.synchronize()
    av.arc_verify_set_timing(True)
    av.arc_verify_kernel_stats(reset=True)
    for _ in range(STEPS):
        fn()
    torch.cuda.synchronize()
    k, ms = av.arc_verify_kernel_stats(reset=True)
    av.arc_verify_set_timing(False)
    return 1e3 * ms / STEPS


av.init(0)
n = 12 * (1 << 22)  # 12 x 16 MiB f32 per array
reg = Region("F", "f32", n, 91, 1e-6, 1e-5, 1024, "f32", n_inject=24)
o, r = reg.slice(device="cuda")
one = av.prepare_batch([(o, r, 1e-6, 1e-5, 1024)])
parts = [(o[k * (n // 12):(k + 1) * (n // 12)], r[k * (n // 12):(k + 1) * (n // 12)], 1e-6, 1e-5, 1024)
         for k in range(12)]
twelve = av.prepare_batch(parts)
print(f"one region  {2 * n * 4 / 2**20:.0f} MiB: kernel {kern(one):7.1f} us")
print(f"12 regions  same bytes : kernel {kern(twelve):7.1f} us")
one0 = av.prepare_batch([(o, r, 1e-6, 1e-5, 0)])
twelve0 = av.prepare_batch([(a, b, x, y, 0) for a, b, x, y, _ in parts])
print(f"count-only: one {kern(one0):7.1f} us, twelve {kern(twelve0):7.1f} us")
regs = synth.c3_regions()
data = [rg.slice(device="cuda") for rg in regs]
c3 = av.prepare_batch([(a, b, rg.abs_tol, rg.rel_tol, rg.max_report) for rg, (a, b) in zip(regs, data)])
nb = sum(2 * a.numel() * a.element_size() for a, _ in data)
print(f"C3 {nb / 2**20:.0f} MiB: kernel {kern(c3):7.1f} us")
av.finalize()

# the same bytes as int32 (no float filter warm-up, no seeding): isolates the
# per-region switch cost from the per-region filter warm-up
av.init(0)
oi, ri = o.view(torch.int32), r.view(torch.int32)
one_i = av.prepare_batch([(oi, ri, 0, 0, 0)])
twelve_i = av.prepare_batch([(oi[k * (n // 12):(k + 1) * (n // 12)], ri[k * (n // 12):(k + 1) * (n // 12)], 0, 0, 0)
                             for k in range(12)])
print(f"int32 count-only: one {kern(one_i):7.1f} us, twelve {kern(twelve_i):7.1f} us")
av.finalize()

# float, out == ref bit for bit (separate buffers): no record-breaking
# elements, so no filter warm-up -- what remains is the per-region switch
# (flush + seeding)
av.init(0)
o2 = r.clone()
one_e = av.prepare_batch([(o2, r, 1e-6, 1e-5, 0)])
twelve_e = av.prepare_batch([(o2[k * (n // 12):(k + 1) * (n // 12)], r[k * (n // 12):(k + 1) * (n // 12)], 1e-6, 1e-5,
                              0) for k in range(12)])
print(f"f32 equal count-only: one {kern(one_e):7.1f} us, twelve {kern(twelve_e):7.1f} us")
av.finalize()
