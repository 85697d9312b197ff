"""GPU parity of the collective (NCCL) fallback path with SEVERAL ranks on one GPU.

Real NCCL refuses two ranks on one device and this pool offers one GPU per job,
so the library's NCCL path (csrc/arcv_shard.cu: local packet, all-gather of
fixed-size packets, merge kernel, grouped broadcasts of the entries beyond a
packet) runs here against tests/fakenccl/fake_nccl.cu -- a stand-in for the
seven NCCL calls it makes (uint8 all-gather / broadcast between processes via
CUDA IPC staging buffers and a shared-memory barrier), loaded through
ARCV_NCCL_LIB.  What is tested is the library's logic (packet sizes, the merge
plan on the GPU, phase-B broadcasts and their index offsets, report placement),
not NCCL itself; the 2-GPU test in test_peer_scale_gpu.py runs real NCCL on a
multi-GPU box.  Every rank bit-exact against the unsharded oracle.
"""
import hashlib
import os
import socket
import struct
import subprocess
import sys

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import synth

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
FAKE_SRC = os.path.join(ROOT, "tests", "fakenccl", "fake_nccl.cu")
FAKE_SO = os.path.join(ROOT, "tests", "fakenccl", "libfakenccl.so")


def _bits(x):
    return struct.unpack("<Q", struct.pack("<d", x))[0]


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _build_fake():
    if not os.path.exists(FAKE_SO) or os.path.getmtime(FAKE_SO) < os.path.getmtime(FAKE_SRC):
        subprocess.run(["/usr/local/cuda/bin/nvcc", "-gencode", "arch=compute_100a,code=sm_100a", "-O2",
                        "-std=c++17", "-shared", "-Xcompiler", "-fPIC", "-o", FAKE_SO, FAKE_SRC, "-lrt"],
                       check=True, capture_output=True)
    return FAKE_SO


def _cases():
    # (name, region, max_report): sparse (fits a 4096-entry packet), dense with
    # contributions beyond a packet (phase-B broadcasts), count only
    return [("C1", synth.C1(), 100), ("C4s", synth.C4(1 << 22), 1 << 20), ("C5", synth.C5(1 << 20), 10000),
            ("C5all", synth.C5(1 << 18), 1 << 20), ("C5cnt", synth.C5(1 << 18), 0)]


def _digest(g):
    b = np.ascontiguousarray(np.asarray(g.report[: g.n_reported])).tobytes()
    return (g.n, g.n_mismatch, _bits(g.max_abs_err), _bits(g.max_rel_err), g.n_reported,
            hashlib.sha256(b).hexdigest())


def _worker(rank, world, port, q, fake):
    sys.path.insert(0, ROOT)
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port), ARCV_NCCL_LIB=fake)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    out = []
    try:
        import paper_conf_ipps_leelv14_b200 as av

        torch.cuda.set_device(0)
        assert av.init_distributed(transport="nccl") == "nccl"
        for name, reg, mr in _cases():
            # ragged shards
            cuts = [0] + [min(reg.n, (r + 1) * reg.n // world + 999 * (r + 1)) for r in range(world - 1)] + [reg.n]
            o, r = reg.slice(cuts[rank], cuts[rank + 1] - cuts[rank], device="cuda")
            for rep in range(2):
                g = av.compare(o, r, reg.abs_tol, reg.rel_tol, mr)
                out.append(((name, rep), _digest(g)))
        av.finalize()
        q.put((rank, out, None))
    except Exception:  # pragma: no cover
        import traceback

        q.put((rank, out, traceback.format_exc()))
    finally:
        dist.destroy_process_group()


@pytest.mark.timeout(900)
@pytest.mark.parametrize("world", [2, 3, 4])
def test_nccl_path_several_ranks_fake_nccl(world):
    import oracle

    oracle.build()
    fake = _build_fake()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q, fake)) for r in range(world)]
    for p in procs:
        p.start()
    res = {}
    try:
        for _ in range(world):
            rank, out, err = q.get(timeout=800)
            assert err is None, f"rank {rank}:\n{err}"
            res[rank] = dict(out)
    finally:
        for p in procs:
            p.join(timeout=120)
            if p.is_alive():
                p.kill()
    for r in range(1, world):
        assert res[r] == res[0]
    for name, reg, mr in _cases():
        o, r = reg.slice()
        e = oracle.compare(o.numpy(), r.numpy(), reg.dtype, reg.abs_tol, reg.rel_tol, mr)
        want = (e.n, e.n_mismatch, _bits(e.max_abs_err), _bits(e.max_rel_err), e.n_reported,
                hashlib.sha256(np.ascontiguousarray(e.report).tobytes()).hexdigest())
        for rep in range(2):
            assert res[0][(name, rep)] == want, (world, name, rep, res[0][(name, rep)][:5], want[:5])
