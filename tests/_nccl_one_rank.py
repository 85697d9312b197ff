"""Run in a subprocess by test_parity_gpu.py: the collective (NCCL) path over a
1-rank communicator, compared with the oracle.  Exercises dlopen of NCCL,
ncclCommInitRank, the packet all-gather, the merge kernel and (max_report > K)
the grouped ncclBroadcast of entries beyond a packet."""
import os
import struct
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import oracle  # noqa: E402
import paper_conf_ipps_leelv14_b200 as av  # noqa: E402
import synth  # noqa: E402


def bits(x):
    return struct.unpack("<Q", struct.pack("<d", x))[0]


def main():
    uid = av.arc_verify_get_unique_id()
    av.init(0, rank=0, nranks=1, nccl_unique_id=uid)
    cases = []
    c1 = synth.C1()
    o, r = c1.slice()
    cases.append((o, r, "f32", 1e-6, 1e-5, 100))
    o5, r5 = synth.C5(1 << 16).slice()
    cases.append((o5, r5, "i32", 0, 0, 10000))  # 10000 > K = 4096: phase-B broadcast
    cases.append((o5, r5, "i32", 0, 0, 0))
    for o, r, dt, at, rt, mr in cases:
        g = av.compare(o.cuda(), r.cuda(), at, rt, mr)
        e = oracle.compare(o.numpy(), r.numpy(), dt, at, rt, mr)
        assert (g.n, g.n_mismatch, g.n_reported) == (e.n, e.n_mismatch, e.n_reported), (g, e)
        assert bits(g.max_abs_err) == bits(e.max_abs_err) and bits(g.max_rel_err) == bits(e.max_rel_err)
        assert np.array_equal(g.report, e.report), dt
    av.finalize()
    print("NCCL-ONE-RANK-OK")


if __name__ == "__main__":
    main()
