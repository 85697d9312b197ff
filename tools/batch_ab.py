"""Diagnostic: where a batched grid's per-region cost comes from (C3 and
twelve equal regions), kernel window per call (library CUDA events):
  * C3 in its listed order, sorted by dtype, and Jacobi first / last;
  * C3 count-only (max_report 0) vs with reports;
  * twelve equal f32 / i32 regions vs one region of the same bytes;
  * the read probe over the C3 bytes (one region of the same size).
  python tools/batch_ab.py [LIB.so]
"""
import os
import sys

sys.path.insert(0, os.getcwd())
if len(sys.argv) > 1:
    os.environ["ARCV_LIB_PATH"] = os.path.abspath(sys.argv[1])
import torch  # noqa: E402

import paper_conf_ipps_leelv14_b200 as av  # noqa: E402
import synth  # noqa: E402
from synth.configs import Region  # noqa: E402

STEPS = int(os.environ.get("AB_STEPS", "20"))
L2 = torch.cuda.get_device_properties(0).L2_cache_size
scratch = torch.empty(2 * L2, dtype=torch.uint8, device="cuda")


def kern(fn, flush=True):
    for _ in range(3):
        fn()
    torch.cuda.synchronize()
    tot = 0.0
    for _ in range(STEPS):
        if flush:
            scratch.fill_(1)
        torch.cuda.synchronize()
        av.arc_verify_set_timing(True)
        av.arc_verify_kernel_stats(reset=True)
        fn()
        torch.cuda.synchronize()
        _k, ms = av.arc_verify_kernel_stats(reset=True)
        av.arc_verify_set_timing(False)
        tot += ms
    return 1e3 * tot / STEPS


av.init(0)
regs = synth.c3_regions()
data = [rg.slice(device="cuda") for rg in regs]
nb = sum(2 * a.numel() * a.element_size() for a, _ in data)


def batch(order, mr=None):
    return av.prepare_batch([(data[k][0], data[k][1], regs[k].abs_tol, regs[k].rel_tol,
                              regs[k].max_report if mr is None else mr) for k in order])


listed = list(range(12))
by_dtype = sorted(listed, key=lambda k: ({"f32": 0, "f64": 1, "i32": 2}[regs[k].dtype], k))
jac = [k for k in listed if regs[k].name == "JACOBI"]
rest = [k for k in listed if regs[k].name != "JACOBI"]
print(f"C3 {nb / 2**20:.1f} MiB, order {[regs[k].name for k in listed]}")
for name, order in (("listed", listed), ("by dtype", by_dtype), ("jacobi first", jac + rest),
                    ("jacobi last", rest + jac)):
    print(f"  {name:13s} report {kern(batch(order)):7.1f} us   count-only {kern(batch(order, 0)):7.1f} us")
big = torch.empty(nb // 2, dtype=torch.uint8, device="cuda")
big2 = torch.empty(nb // 2, dtype=torch.uint8, device="cuda")
print(f"  read probe over the same bytes: {2 * (nb // 2) / av.arc_verify_probe_read(big.data_ptr(), big2.data_ptr(), nb // 2, 20) / 1e3:7.1f} us")
del big, big2

for dt in ("f32", "i32"):
    n = 12 * (1 << 22)
    reg = Region("F", dt, n, 91, 1e-6 if dt == "f32" else 0, 1e-5 if dt == "f32" else 0, 1024, dt, n_inject=24)
    o, r = reg.slice(device="cuda")
    at, rt = (1e-6, 1e-5) if dt == "f32" else (0, 0)
    one = av.prepare_batch([(o, r, at, rt, 1024)])
    parts = [(o[k * (n // 12):(k + 1) * (n // 12)], r[k * (n // 12):(k + 1) * (n // 12)], at, rt, 1024)
             for k in range(12)]
    print(f"{dt}: one region {2 * n * 4 / 2**20:.0f} MiB {kern(one, False):7.1f} us | twelve equal {kern(av.prepare_batch(parts), False):7.1f} us"
          f" | count-only one {kern(av.prepare_batch([(o, r, at, rt, 0)]), False):7.1f} twelve "
          f"{kern(av.prepare_batch([(a, b, x, y, 0) for a, b, x, y, _ in parts]), False):7.1f} us")
av.finalize()
