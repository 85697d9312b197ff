"""Sharded (N>1) path on CPU: world_size-2 process group over gloo.

The GPU kernels cannot run here, so each rank computes its shard's partial
result with the oracle (test infrastructure) and the ranks exchange them over
a real torch.distributed group exactly as the library's collective does
(headers all-gathered first, then report entries): the merge plan comes from
the library's own host function arc_verify_merge_plan (C ABI, no GPU).  Both
ranks must assemble the same global result, equal to the unsharded oracle.
"""
import os
import socket
import struct
import sys

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _bits(x):
    return struct.unpack("<Q", struct.pack("<d", x))[0]


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, max_report, cuts, q):
    sys.path.insert(0, ROOT)
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import oracle
        import paper_conf_ipps_leelv14_b200 as av
        import synth

        c1 = synth.C1()
        a, b = cuts[rank], cuts[rank + 1]
        out, ref = c1.slice(a, b - a)  # each rank generates only its shard
        part = oracle.compare(out.numpy(), ref.numpy(), "f32", c1.abs_tol, c1.rel_tol, max_report)
        # 1) all-gather the 32-byte headers
        s64 = lambda v: v - (1 << 64) if v >= (1 << 63) else v  # noqa: E731
        hdr = torch.tensor([part.n, part.n_mismatch, s64(_bits(part.max_abs_err)), s64(_bits(part.max_rel_err))],
                           dtype=torch.int64)
        hdrs = [torch.zeros(4, dtype=torch.int64) for _ in range(world)]
        dist.all_gather(hdrs, hdr)
        headers = [tuple(int(v) & ((1 << 64) - 1) for v in h.tolist()) for h in hdrs]
        plan, glob = av.arc_verify_merge_plan(headers, max_report)
        # 2) exchange the report entries each rank contributes (variable length:
        #    pad to the max contribution, like the library's fixed-size packets)
        K = max(1, max(p[2] for p in plan))
        mine = np.zeros(K, dtype=av.REPORT_DTYPE)
        c = plan[rank][2]
        mine[:c] = part.report[:c]
        buf = torch.from_numpy(mine.view(np.int64).copy())
        bufs = [torch.zeros_like(buf) for _ in range(world)]
        dist.all_gather(bufs, buf)
        final = []
        for r in range(world):
            ent = bufs[r].numpy().view(av.REPORT_DTYPE)[: plan[r][2]].copy()
            ent["index"] += np.uint64(plan[r][0])
            final.append(ent)
        final = np.concatenate(final)
        q.put((rank, glob, final.tobytes()))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("max_report", [0, 7, 45, 1000])
def test_world2_gloo_merge_equals_unsharded(max_report):
    import oracle
    import paper_conf_ipps_leelv14_b200  # noqa: F401  (the .so must load on CPU)
    import synth

    c1 = synth.C1()
    n = c1.n
    cuts = [0, 400_009, n]  # ragged split; C1's planted mismatches fall on both sides
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, max_report, cuts, q)) for r in range(2)]
    for p in procs:
        p.start()
    got = [q.get(timeout=180) for _ in range(2)]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    out, ref = c1.slice()
    full = oracle.compare(out.numpy(), ref.numpy(), "f32", c1.abs_tol, c1.rel_tol, max_report)
    for rank, glob, rep in got:
        assert glob[0] == n and glob[1] == full.n_mismatch
        assert glob[2] == _bits(full.max_abs_err) and glob[3] == _bits(full.max_rel_err)
        assert rep == full.report.tobytes(), rank
    assert got[0][2] == got[1][2]
