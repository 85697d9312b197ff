"""Diagnostic: report vs count-only (max_report = 0) kernel time at one size,
interleaved A/B/A/B so that clock and power drift hit both arms alike.
size_sweep.py measures count-only right after the report arm at each size; at
2^29 fp64 its count-only figure came out above the report arm's on three boxes.
  python tools/count_only_ab.py [log2 n] [rounds]
"""
import os
import sys

sys.path.insert(0, os.getcwd())
import torch

import paper_conf_ipps_leelv14_b200 as av
import synth

LG = int(sys.argv[1]) if len(sys.argv) > 1 else 29
ROUNDS = int(sys.argv[2]) if len(sys.argv) > 2 else 6
STEPS = 20
REP = torch.empty(24 * (1 << 20), dtype=torch.uint8, pin_memory=True).numpy().view(av.REPORT_DTYPE)

av.init(0)
reg = synth.C4(1 << LG)
o, r = reg.slice(device="cuda")
torch.cuda.synchronize()
steps = {mr: av.prepare(o, r, reg.abs_tol, reg.rel_tol, mr, report=REP) for mr in (1 << 20, 0)}
for s in steps.values():
    for _ in range(5):
        s()
torch.cuda.synchronize()
res = {mr: [] for mr in steps}
for rnd in range(ROUNDS):
    order = (1 << 20, 0) if rnd % 2 == 0 else (0, 1 << 20)
    for mr in order:
        av.arc_verify_set_timing(True)
        av.arc_verify_kernel_stats(reset=True)
        for _ in range(STEPS):
            steps[mr]()
        torch.cuda.synchronize()
        k, kms = av.arc_verify_kernel_stats(reset=True)
        av.arc_verify_set_timing(False)
        res[mr].append(1e3 * kms / k)
nb = 2 * 8 * (1 << LG)
for mr, v in res.items():
    v = sorted(v)
    print(f"f64 2^{LG} max_report={mr:8d}: kernel us min {v[0]:8.1f} median {v[len(v)//2]:8.1f} "
          f"max {v[-1]:8.1f}  (median {nb / v[len(v)//2] / 1e3:6.0f} GB/s)  all {[round(x, 1) for x in res[mr]]}")
av.finalize()
