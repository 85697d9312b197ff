"""Fixed cost of the sharded exchange on one GPU (p = 1): per-call wall time of
  local   -- arc_verify_compare, single-GPU path
  peer    -- the same call through the peer-memory exchange (window + exchange
             kernel; the flag round trip goes to the own window)
  nccl    -- the same call through the NCCL path over a 1-rank communicator
Each mode runs in its own process (one library context per process).
  python tools/exchange_overhead.py            # all modes
"""
import json
import os
import subprocess
import sys
import time

MODES = ("local", "peer", "nccl")


def child(mode):
    sys.path.insert(0, os.getcwd())
    import numpy as np
    import torch

    import paper_conf_ipps_leelv14_b200 as av
    import synth

    torch.cuda.set_device(0)
    if mode == "nccl":
        av.init(0, rank=0, nranks=1, nccl_unique_id=av.arc_verify_get_unique_id())
    else:
        av.init(0)
        if mode == "peer":
            av.arc_verify_peer_open([av.arc_verify_peer_export(1 << 20)])
    rep = torch.empty(24 * (1 << 20), dtype=torch.uint8, pin_memory=True).numpy().view(av.REPORT_DTYPE)
    res = {}
    cases = [("C1 f32 2^20 (45 mism.)", synth.C1(), 1 << 20),
             ("C4 f64 2^24 (sparse)", synth.C4(1 << 24), 1 << 20),
             ("C4 f64 2^29 (bench)", synth.C4(), 1 << 20)]
    for name, reg, mr in cases:
        o, r = reg.slice(device="cuda")
        call = av.prepare(o, r, reg.abs_tol, reg.rel_tol, mr, report=rep)
        for _ in range(5):
            g = call()
        torch.cuda.synchronize()
        steps = 50
        t0 = time.perf_counter()
        for _ in range(steps):
            g = call()
        dt = (time.perf_counter() - t0) / steps
        res[name] = {"us_per_call": round(dt * 1e6, 1), "n_mismatch": g.n_mismatch,
                     "report_head": [int(x) for x in np.asarray(g.report["index"][:3])]}
        del o, r, call
        torch.cuda.empty_cache()
    av.finalize()
    print("RESULT " + json.dumps(res), flush=True)


def main():
    if len(sys.argv) > 2 and sys.argv[1] == "--child":
        return child(sys.argv[2])
    out = {}
    for m in MODES:
        p = subprocess.run([sys.executable, __file__, "--child", m], capture_output=True, text=True, timeout=600)
        line = [x for x in p.stdout.splitlines() if x.startswith("RESULT ")]
        out[m] = json.loads(line[0][7:]) if line else {"error": (p.stderr or p.stdout)[-800:]}
    for m in MODES:
        print(m, json.dumps(out[m]))


if __name__ == "__main__":
    main()
