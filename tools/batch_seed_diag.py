import os, sys, ctypes
sys.path.insert(0, os.getcwd())
import torch
import paper_conf_ipps_leelv14_b200 as av
from synth.configs import Region
libs = sys.argv[1:]
n = 12 * (1 << 22)
reg = Region("F", "f32", n, 91, 1e-6, 1e-5, 1024, "f32", n_inject=24)
o, r = reg.slice(device="cuda"); o2 = r.clone()
m = n // 12
stream = torch.cuda.current_stream().cuda_stream
for path in libs:
    lib = ctypes.CDLL(os.path.abspath(path))
    lib.arc_verify_init.argtypes = [ctypes.POINTER(av.arc_verify_opts_t)]
    lib.arc_verify_batch.argtypes = [ctypes.POINTER(av.arc_verify_region_t), ctypes.c_size_t, ctypes.POINTER(av.arc_verify_result_t)]
    lib.arc_verify_kernel_stats.argtypes = [ctypes.POINTER(ctypes.c_uint64), ctypes.POINTER(ctypes.c_double), ctypes.c_int]
    opts = av.arc_verify_opts_t(0, stream or 1, 0, 1, None)
    assert lib.arc_verify_init(ctypes.byref(opts)) == 0
    for name, a, b in (("noisy", o, r), ("equal", o2, r)):
        for k in (1, 12):
            R = (av.arc_verify_region_t * k)(); res = (av.arc_verify_result_t * k)()
            for i in range(k):
                sz = n // k
                R[i].out = a[i*sz:(i+1)*sz].data_ptr(); R[i].ref = b[i*sz:(i+1)*sz].data_ptr(); R[i].n = sz
                R[i].dtype = 0; R[i].abs_tol = 1e-6; R[i].rel_tol = 1e-5; R[i].max_report = 0
            for _ in range(3): lib.arc_verify_batch(R, k, res)
            torch.cuda.synchronize(); lib.arc_verify_set_timing(1)
            nn, ms = ctypes.c_uint64(), ctypes.c_double(); lib.arc_verify_kernel_stats(ctypes.byref(nn), ctypes.byref(ms), 1)
            for _ in range(20): lib.arc_verify_batch(R, k, res)
            lib.arc_verify_kernel_stats(ctypes.byref(nn), ctypes.byref(ms), 1); lib.arc_verify_set_timing(0)
            print(f"{os.path.basename(path):14s} {name:6s} regions={k:2d} count-only kernel {1e3*ms.value/nn.value:7.1f} us", flush=True)
    lib.arc_verify_finalize()
