"""Diagnostic: fixed per-launch cost of the compare vs the read probe."""
import os, sys, time
sys.path.insert(0, os.getcwd())
import torch, synth
import paper_conf_ipps_leelv14_b200 as av
REP = torch.empty(24 * (1 << 20), dtype=torch.uint8, pin_memory=True).numpy().view(av.REPORT_DTYPE)
def kt(out, ref, at, rt, mr, steps=30):
    for _ in range(3): av.compare(out, ref, at, rt, mr, report=REP)
    torch.cuda.synchronize()
    av.arc_verify_set_timing(True); av.arc_verify_kernel_stats(reset=True)
    for _ in range(steps): av.compare(out, ref, at, rt, mr, report=REP)
    torch.cuda.synchronize()
    n, ms = av.arc_verify_kernel_stats(reset=True); av.arc_verify_set_timing(False)
    return 1e3 * ms / n
av.init(0)
c2 = synth.C2("A"); o, r = c2.slice(device="cuda")
nb = o.numel() * 4
print("probe C2-size", 2 * nb / av.arc_verify_probe_read(o.data_ptr(), r.data_ptr(), nb, 30) / 1e3, "us")
print("compare out==ref f32", kt(o, o, 0.0, 1e-5, 0), "us")
print("compare C2A f32", kt(o, r, 0.0, 1e-5, 0), "us")
print("compare C2A as i32", kt(o.view(torch.int32), r.view(torch.int32), 0, 0, 0), "us (mismatching everywhere)")
print("compare out==ref as i32", kt(o.view(torch.int32), o.view(torch.int32), 0, 0, 0), "us")
print("compare out==ref as u8", kt(o.view(torch.uint8), o.view(torch.uint8), 0, 0, 0), "us")
for n in (1 << 16, 1 << 20, 1 << 22):
    x = o[:n]; y = r[:n]
    print(f"n={n} probe", 2 * n * 4 / av.arc_verify_probe_read(x.data_ptr(), y.data_ptr(), n * 4, 50) / 1e3, "us;",
          "compare", kt(x, y, 0.0, 1e-5, 0), "us")
av.finalize()
