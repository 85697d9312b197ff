"""Diagnostic: per-call host overhead (python binding vs raw ctypes vs kernel events)."""
import os, sys, time, ctypes
sys.path.insert(0, os.getcwd())
import torch, synth
import paper_conf_ipps_leelv14_b200 as av
av.init(0)
for n, label in ((1 << 20, "C1-size f32"), (1 << 26, "C2-size f32")):
    reg = synth.configs.Region("F", "f32", n, 5, 1e-6, 1e-5, 1 << 20, "f32")
    o, r = reg.slice(device="cuda")
    REP = torch.empty(24 * (1 << 20), dtype=torch.uint8, pin_memory=True).numpy().view(av.REPORT_DTYPE)
    for mr in (0, 1 << 20):
        for _ in range(5): av.compare(o, r, 1e-6, 1e-5, mr, report=REP)
        torch.cuda.synchronize()
        av.arc_verify_set_timing(True); av.arc_verify_kernel_stats(reset=True)
        N = 200
        t0 = time.perf_counter()
        for _ in range(N): av.compare(o, r, 1e-6, 1e-5, mr, report=REP)
        t1 = time.perf_counter()
        nl, ms = av.arc_verify_kernel_stats(reset=True); av.arc_verify_set_timing(False)
        res = av.arc_verify_result_t(); res.report = REP.ctypes.data
        po, pr = o.data_ptr(), r.data_ptr()
        f = av._lib.arc_verify_compare; br = ctypes.byref(res)
        t2 = time.perf_counter()
        for _ in range(N): f(po, pr, n, 0, 1e-6, 1e-5, mr, br)
        t3 = time.perf_counter()
        call = av.prepare(o, r, 1e-6, 1e-5, mr, report=REP)
        t4 = time.perf_counter()
        for _ in range(N): call()
        t5 = time.perf_counter()
        print(f"{label} mr={mr}: python compare {1e6*(t1-t0)/N:.1f} us/call, prepared {1e6*(t5-t4)/N:.1f}, "
              f"raw ctypes {1e6*(t3-t2)/N:.1f} us/call, kernels {1e3*ms/nl:.1f} us", flush=True)
av.finalize()
