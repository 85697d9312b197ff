"""Diagnostic: read-probe vs compare throughput over sizes and dtypes."""
import os, sys, time
sys.path.insert(0, os.getcwd())
import torch, synth
import paper_conf_ipps_leelv14_b200 as av
from synth.configs import Region
REP = torch.empty(24 * (1 << 20), dtype=torch.uint8, pin_memory=True).numpy().view(av.REPORT_DTYPE)
def run(label, out, ref, at, rt, mr, steps=20):
    for _ in range(3): av.compare(out, ref, at, rt, mr, report=REP)
    torch.cuda.synchronize()
    av.arc_verify_set_timing(True); av.arc_verify_kernel_stats(reset=True)
    for _ in range(steps): r = av.compare(out, ref, at, rt, mr, report=REP)
    torch.cuda.synchronize()
    n, ms = av.arc_verify_kernel_stats(reset=True); av.arc_verify_set_timing(False)
    b = 2 * out.numel() * out.element_size()
    print(f"{label:40s} kernel {b/(ms/n/1e3)/1e9:8.1f} GB/s  ({ms/n*1e3:8.1f} us) mism={r.n_mismatch}", flush=True)
av.init(0)
for nb in (1 << 26, 1 << 28, 1 << 30, 1 << 32):
    a = torch.empty(nb, dtype=torch.uint8, device="cuda"); b = torch.empty(nb, dtype=torch.uint8, device="cuda")
    print(f"probe {nb>>20} MiB/array: {av.arc_verify_probe_read(a.data_ptr(), b.data_ptr(), nb, 10):.1f} GB/s", flush=True)
    del a, b
for n in (1 << 26, 1 << 28, 1 << 29):
    reg = Region("F", "f32", n, 77, 1e-6, 1e-5, 1 << 20, "f32")
    o, r = reg.slice(device="cuda")
    run(f"f32 uniform n=2^{n.bit_length()-1} mr=0", o, r, 1e-6, 1e-5, 0)
    run(f"f32 uniform n=2^{n.bit_length()-1} mr=2^20", o, r, 1e-6, 1e-5, 1 << 20)
    del o, r
for n in (1 << 28,):
    reg = Region("I", "i32", n, 78, 0, 0, 1 << 20, "i32")
    o, r = reg.slice(device="cuda")
    run(f"i32 n=2^28 clean mr=2^20", o, r, 0, 0, 1 << 20)
    run(f"u8 view n=2^30 clean mr=2^20", o.view(torch.uint8), r.view(torch.uint8), 0, 0, 1 << 20)
    run(f"i64 view n=2^27 clean mr=2^20", o.view(torch.int64), r.view(torch.int64), 0, 0, 1 << 20)
c2 = synth.C2("A"); o, r = c2.slice(device="cuda")
run("C2A f32 mr=2^20", o, r, 0.0, 1e-5, 1 << 20)
run("C2A f32 mr=0", o, r, 0.0, 1e-5, 0)
av.finalize()
