"""GPU parity of the sharded path at the north_star shapes (BASELINE.json
configs[3] / configs[4]), over the peer-memory exchange.

World sizes 2, 3, 4 and 8 run as separate processes on ONE GPU (each rank its
own CUDA context; the windows are mapped through CUDA IPC; the exchange waits on
flags stored by other processes) -- the same code that runs across the GPUs of
an NVSwitch box, only the link differs (include/arc_verify.h: ranks may share a
device).  torch.distributed (gloo) carries only the 64-byte window handles.

  * C5 shape: int32, out = ref ^ (i & 1) (50 % mismatches), n = 2^24,
    max_report = 2^20 with a window capacity of 2^20: rank 0 holds the first
    2^24 / p elements and contributes every one of the 2^20 global report
    entries at p <= 8 (the compaction / exchange worst case);
  * C4 shape: fp64, 2^26 elements PER RANK (the p = 8 shard of the 4 GiB
    config), 512 injected + 4 NaN pairs, max_report 2^20.

Report buffers: pageable host memory, pinned host memory and device memory.
Every rank must hold the identical global result, bit-exact against the
unsharded oracle (compare_threads: the oracle on contiguous chunks merged by
merge_shards, pinned equal to the sequential oracle in tests/test_oracle.py).
Two more tests need one GPU per rank and skip on a one-GPU box: the peer exchange
across 2 / 4 / 8 physical GPUs, and the NCCL transport with two ranks on two GPUs
(NCCL refuses two ranks on one device).
"""
import hashlib
import os
import socket
import struct
import sys

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import synth

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
C5_N = 1 << 24
C4_PER_RANK = 1 << 26
MR = 1 << 20


def _bits(x):
    return struct.unpack("<Q", struct.pack("<d", x))[0]


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _digest(g, av):
    rep = g.report
    if isinstance(rep, torch.Tensor):
        rep = rep[: 24 * g.n_reported].cpu().numpy().view(av.REPORT_DTYPE)
    b = np.ascontiguousarray(np.asarray(rep[: g.n_reported])).tobytes()
    return (g.n, g.n_mismatch, _bits(g.max_abs_err), _bits(g.max_rel_err), g.n_reported,
            hashlib.sha256(b).hexdigest())


def _cases(world):
    return [("C5", synth.C5(C5_N), "i32"), ("C4", synth.C4(C4_PER_RANK * world), "f64")]


def _worker(rank, world, port, q, transport, device):
    sys.path.insert(0, ROOT)
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    out = []
    try:
        import paper_conf_ipps_leelv14_b200 as av

        torch.cuda.set_device(device(rank))
        got = av.init_distributed(transport=transport, max_report_cap=MR)
        assert got == transport, got
        pinned = torch.empty(24 * MR, dtype=torch.uint8, pin_memory=True).numpy().view(av.REPORT_DTYPE)
        dev_rep = torch.empty(24 * MR, dtype=torch.uint8, device="cuda")
        cases = {name: reg for name, reg, _dt in _cases(world)}
        # C5 (dense: ring forwarding at p >= 3), C4 (sparse: pull), C5 again
        # (the ring's per-call chunk counters after a pull-mode call)
        for name, reps in (("C5", range(4)), ("C4", range(4)), ("C5", range(4, 6))):
            reg = cases[name]
            a, b = rank * reg.n // world, (rank + 1) * reg.n // world
            o, r = reg.slice(a, b - a, device="cuda")
            av.arc_verify_peer_stats(reset=True)
            for rep in reps:  # consecutive calls alternate the window parity
                buf = (None, pinned, dev_rep, pinned, dev_rep, None)[rep]
                g = av.compare(o, r, reg.abs_tol, reg.rel_tol, reg.max_report, report=buf)
                out.append(((name, rep), _digest(g, av)))
            pulled, forwarded = av.arc_verify_peer_stats()
            out.append(((name, "bytes", reps[0]), (pulled // len(reps), forwarded // len(reps))))
            del o, r
            torch.cuda.empty_cache()
        av.finalize()
        q.put((rank, out, None))
    except Exception:  # pragma: no cover - reported to the parent
        import traceback

        q.put((rank, out, traceback.format_exc()))
    finally:
        dist.destroy_process_group()


def _expected(world):
    """The unsharded oracle on the same seeded arrays (generated on the GPU, read back)."""
    import oracle

    oracle.build()
    want = {}
    for name, reg, dt in _cases(world):
        o, r = reg.slice(device="cuda")
        o, r = o.cpu().numpy(), r.cpu().numpy()
        e = oracle.compare_threads(o, r, dt, reg.abs_tol, reg.rel_tol, reg.max_report)
        want[name] = (e.n, e.n_mismatch, _bits(e.max_abs_err), _bits(e.max_rel_err), e.n_reported,
                      hashlib.sha256(np.ascontiguousarray(e.report).tobytes()).hexdigest())
        # closed forms of the generator, independent of the oracle
        if name == "C5":
            assert e.n_mismatch == C5_N // 2 and e.n_reported == MR and e.max_abs_err == 1.0
            assert np.array_equal(e.report["index"], np.arange(1, 2 * MR, 2, dtype=np.uint64))
        else:
            assert e.n_mismatch == 516 and list(e.report["index"]) == reg.planted()
        del o, r
        torch.cuda.empty_cache()
    return want


def _run(world, transport, device, timeout=900):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q, transport, device)) for r in range(world)]
    for p in procs:
        p.start()
    res = {}
    try:
        for _ in range(world):
            rank, out, err = q.get(timeout=timeout)
            assert err is None, f"rank {rank}:\n{err}"
            res[rank] = dict(out)
    finally:
        for p in procs:
            p.join(timeout=120)
            if p.is_alive():
                p.kill()
    for p in procs:
        assert p.exitcode == 0
    return res


def _results(d):
    """The global results (identical on every rank); per-rank byte counters excluded."""
    return {k: v for k, v in d.items() if "bytes" not in k}


def _on_gpu0(rank):
    return 0


def _own_gpu(rank):
    return rank


@pytest.mark.timeout(1500)
@pytest.mark.parametrize("world", [2, 3, 4, 8])
def test_sharded_north_star_shapes_peer(world):
    res = _run(world, "peer", _on_gpu0)
    for r in range(1, world):
        assert _results(res[r]) == _results(res[0]), f"rank {r} differs from rank 0"
    want = _expected(world)
    for name, reps in (("C5", range(6)), ("C4", range(4))):
        for rep in reps:
            assert res[0][(name, rep)] == want[name], (world, name, rep, res[0][(name, rep)], want[name])
    # bytes read from peer windows per call (measured by the exchange kernels):
    # C5's 2^20 entries all belong to rank 0; with ring forwarding (p >= 3)
    # rank 1 pulls them from rank 0 and rank k >= 2 from rank k - 1, so every
    # window is read once; at p = 2 rank 1 pulls them from rank 0
    rep_bytes = 24 * MR
    for first in (0, 4):
        per_rank = [res[r][("C5", "bytes", first)] for r in range(world)]
        assert per_rank[0] == (0, 0), per_rank
        assert per_rank[1] == (rep_bytes, 0), per_rank
        for r in range(2, world):
            assert per_rank[r] == (0, rep_bytes), (r, per_rank)
    # C4 (516 entries, pull): each rank reads the other ranks' contributions once


@pytest.mark.timeout(1500)
@pytest.mark.parametrize("world", [2, 4, 8])
def test_sharded_north_star_shapes_peer_own_gpus(world):
    """The peer exchange with one rank per physical GPU (windows mapped over NVLink /
    NVSwitch instead of within one device); skips unless `world` GPUs are visible."""
    if torch.cuda.device_count() < world:
        pytest.skip(f"needs {world} GPUs (one per rank); {torch.cuda.device_count()} visible")
    res = _run(world, "peer", _own_gpu)
    for r in range(1, world):
        assert _results(res[r]) == _results(res[0]), f"rank {r} differs from rank 0"
    want = _expected(world)
    for name, reps in (("C5", range(6)), ("C4", range(4))):
        for rep in reps:
            assert res[0][(name, rep)] == want[name], (world, name, rep)


@pytest.mark.timeout(1500)
@pytest.mark.skipif(torch.cuda.device_count() < 2, reason="NCCL needs one GPU per rank (2 GPUs)")
def test_sharded_north_star_shapes_nccl_two_gpus():
    """The NCCL fallback (all-gather of packets, merge kernel, grouped broadcast of
    the entries beyond a packet: C5's 2^20-entry report) across two real GPUs."""
    res = _run(2, "nccl", _own_gpu)
    assert _results(res[1]) == _results(res[0])
    want = _expected(2)
    for name, reps in (("C5", range(6)), ("C4", range(4))):
        for rep in reps:
            assert res[0][(name, rep)] == want[name], (name, rep)


def _multi_worker(rank, world, port, q, n, mr):
    sys.path.insert(0, ROOT)
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    out = []
    try:
        import paper_conf_ipps_leelv14_b200 as av

        torch.cuda.set_device(0)
        assert av.init_distributed(transport="peer", max_report_cap=MR) == "peer"
        reg = synth.C5(n)
        # ragged shards: rank r gets a slightly different length
        cuts = [0] + [min(n, (r + 1) * n // world + 777 * (r + 1)) for r in range(world - 1)] + [n]
        o, r = reg.slice(cuts[rank], cuts[rank + 1] - cuts[rank], device="cuda")
        dev_rep = torch.empty(24 * MR, dtype=torch.uint8, device="cuda")
        av.arc_verify_peer_stats(reset=True)
        for rep in range(3):
            g = av.compare(o, r, 0, 0, mr, report=(None, dev_rep, None)[rep])
            out.append(((rep,), _digest(g, av)))
        out.append((("bytes",), av.arc_verify_peer_stats()))
        av.finalize()
        q.put((rank, out, None))
    except Exception:  # pragma: no cover
        import traceback

        q.put((rank, out, traceback.format_exc()))
    finally:
        dist.destroy_process_group()


@pytest.mark.timeout(900)
@pytest.mark.parametrize("world", [3, 5])
def test_ring_many_contributors_ragged(world):
    """Ring forwarding with several contributing ranks: C5-shaped int32 (50 % mismatches)
    over n = 2^21 + 12345 elements in ragged shards and max_report = 2^20 - 7, so most ranks
    contribute, contributions are not multiples of the 384 KB chunk and the last one is
    truncated.  Every rank bit-exact against the unsharded oracle; the bytes each rank read
    from peer windows equal (p - 1) x the report -- no window is read twice per call."""
    import oracle

    oracle.build()
    n, mr = (1 << 21) + 12345, MR - 7
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_multi_worker, args=(r, world, port, q, n, mr)) for r in range(world)]
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
    o, r = synth.C5(n).slice()
    e = oracle.compare(o.numpy(), r.numpy(), "i32", 0, 0, mr)
    want = (e.n, e.n_mismatch, _bits(e.max_abs_err), _bits(e.max_rel_err), e.n_reported,
            hashlib.sha256(np.ascontiguousarray(e.report).tobytes()).hexdigest())
    assert e.n_reported == mr
    for rank in range(world):
        for rep in range(3):
            assert res[rank][(rep,)] == want, (world, rank, rep)
    # each rank receives the report entries it does not own exactly once per call
    # (ring: from its predecessor; its own from its own window, locally)
    tot = sum(sum(res[rank][("bytes",)]) for rank in range(world))
    assert tot == 3 * (world - 1) * 24 * mr, (tot, [res[k][("bytes",)] for k in range(world)])
