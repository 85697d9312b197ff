"""GPU parity of the sharded path over the peer-memory exchange (arcv_peer.cu).

World-size 2 and 3 process groups run on ONE GPU: every rank is its own process
with its own CUDA context, so the peer windows really are mapped through CUDA
IPC and the exchange kernel really waits on flags stored by other processes --
the same code that runs across the GPUs of an NVSwitch box (only the link
differs).  torch.distributed (gloo) carries only the 64-byte window handles.
Every rank must receive the identical global result, bit-exact against the
unsharded CPU oracle, over several consecutive calls (both window parities).
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

import synth

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _bits(x):
    return struct.unpack("<Q", struct.pack("<d", x))[0]


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _cases():
    """(name, region factory, cuts as fractions or absolute, max_report list)."""
    return [
        ("C1", lambda: synth.C1(), [1e-6, 1e-5], "f32"),
        ("C4s", lambda: synth.C4(1 << 20), [1e-6, 1e-5], "f64"),
        ("C5s", lambda: synth.C5(1 << 16), [0.0, 0.0], "i32"),
    ]


def _cuts(n, world, kind):
    if kind == "even":
        return [r * n // world for r in range(world + 1)]
    if kind == "ragged":
        c = [0] + [min(n, (r + 1) * n // world + 4097 * (r + 1)) for r in range(world - 1)] + [n]
        return c
    if kind == "empty0":  # rank 0 holds nothing
        return [0, 0] + [r * n // (world - 1) for r in range(1, world)]
    raise ValueError(kind)


def _worker(rank, world, port, q):
    sys.path.insert(0, ROOT)
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    out = []
    try:
        import paper_conf_ipps_leelv14_b200 as av

        torch.cuda.set_device(0)
        assert av.init_distributed(transport="peer", max_report_cap=1 << 14) == "peer"
        # report buffers: pageable (HBM staging + D2H), pinned (a sparse global report is
        # written by the exchange kernel straight over PCIe), device memory
        pinned = torch.empty(24 << 14, dtype=torch.uint8, pin_memory=True).numpy().view(av.REPORT_DTYPE)
        dev_rep = torch.empty(24 << 14, dtype=torch.uint8, device="cuda")
        for name, mk, (at, rt), dt in _cases():
            reg = mk()
            for kind in ("even", "ragged", "empty0"):
                cuts = _cuts(reg.n, world, kind)
                a, b = cuts[rank], cuts[rank + 1]
                o, r = reg.slice(a, b - a, device="cuda")
                for mr in (0, 7, 100, 1 << 14):
                    for rep in range(3):  # consecutive calls alternate the window parity
                        buf = (None, pinned, dev_rep)[rep]
                        g = av.compare(o, r, at, rt, mr, report=buf)
                        entries = g.report
                        if isinstance(entries, torch.Tensor):
                            entries = entries.cpu().numpy().view(av.REPORT_DTYPE)[: g.n_reported]
                        out.append(((name, kind, mr, rep), (g.n, g.n_mismatch, _bits(g.max_abs_err),
                                                            _bits(g.max_rel_err), g.n_reported,
                                                            np.array(entries[: g.n_reported]).tobytes())))
        # a report larger than the window with no NCCL communicator: refused, not wrong
        try:
            av.compare(o, r, 0, 0, (1 << 14) + 1)
            out.append((("oversize",), "accepted"))
        except av.ArcVerifyError as e:
            out.append((("oversize",), "refused" if e.status == av.ARC_E_UNSUPPORTED else str(e)))
        av.finalize()
        q.put((rank, out, None))
    except Exception as e:  # pragma: no cover - reported to the parent
        import traceback

        q.put((rank, out, traceback.format_exc()))
    finally:
        dist.destroy_process_group()


@pytest.mark.timeout(600)
@pytest.mark.parametrize("world,fused", [(2, "1"), (3, "1"), (2, "0")])
def test_peer_exchange_matches_unsharded_oracle(world, fused, monkeypatch):
    """fused = 1: the exchange runs in K1's tail (one kernel per call); 0: the separate
    exchange kernel (also what empty shards use)."""
    import oracle

    oracle.build()
    monkeypatch.setenv("ARCV_FUSED_EXCHANGE", fused)  # inherited by the spawned ranks
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = {}
    for _ in range(world):
        rank, out, err = q.get(timeout=540)
        assert err is None, f"rank {rank}:\n{err}"
        res[rank] = dict(out)
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    # every rank holds the identical global result
    for r in range(1, world):
        assert res[r] == res[0]
    assert res[0][("oversize",)] == "refused"
    # ... equal to the unsharded oracle
    for name, mk, (at, rt), dt in _cases():
        reg = mk()
        o, r = reg.slice()
        for mr in (0, 7, 100, 1 << 14):
            e = oracle.compare(o.numpy(), r.numpy(), dt, at, rt, mr)
            want = (e.n, e.n_mismatch, _bits(e.max_abs_err), _bits(e.max_rel_err), e.n_reported,
                    np.ascontiguousarray(e.report).tobytes())
            for kind in ("even", "ragged", "empty0"):
                for rep in range(3):
                    got = res[0][(name, kind, mr, rep)]
                    assert got[:5] == want[:5], (name, kind, mr, rep, got[:5], want[:5])
                    assert got[5] == want[5], (name, kind, mr, rep)


def _stress_worker(rank, world, port, q, calls):
    sys.path.insert(0, ROOT)
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import paper_conf_ipps_leelv14_b200 as av

        torch.cuda.set_device(0)
        assert av.init_distributed(transport="peer", max_report_cap=1 << 12) == "peer"
        regs = [synth.C4(1 << 20), synth.C1()]
        shards = []
        for reg in regs:
            a, b = rank * reg.n // world, (rank + 1) * reg.n // world
            shards.append(reg.slice(a, b - a, device="cuda"))
        pinned = torch.empty(24 << 12, dtype=torch.uint8, pin_memory=True).numpy().view(av.REPORT_DTYPE)
        digest = []
        for it in range(calls):
            k = it % 2
            reg, (o, r) = regs[k], shards[k]
            mr = (7, 4096, 100)[it % 3]
            g = av.compare(o, r, reg.abs_tol, reg.rel_tol, mr, report=pinned if it % 5 else None)
            digest.append((k, mr, g.n_mismatch, g.n_reported,
                           tuple(int(i) for i in np.asarray(g.report["index"][: g.n_reported]))))
        av.finalize()
        q.put((rank, digest, None))
    except Exception:  # pragma: no cover
        import traceback

        q.put((rank, None, traceback.format_exc()))
    finally:
        dist.destroy_process_group()


@pytest.mark.timeout(600)
def test_peer_exchange_many_calls():
    """300 back-to-back sharded calls (world 2, exchange fused into K1): window parities,
    sequence numbers and the exchange counters stay in step; every call equals the
    generator's closed form on every rank."""
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    calls = 300
    procs = [ctx.Process(target=_stress_worker, args=(r, 2, port, q, calls)) for r in range(2)]
    for p in procs:
        p.start()
    res = {}
    for _ in range(2):
        rank, digest, err = q.get(timeout=540)
        assert err is None, f"rank {rank}:\n{err}"
        res[rank] = digest
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    assert res[0] == res[1]
    planted = [synth.C4(1 << 20).planted(), synth.C1().planted()]
    for k, mr, n_mis, n_rep, head in res[0]:
        assert n_mis == len(planted[k]) and n_rep == min(n_mis, mr)
        assert list(head) == planted[k][:n_rep]


def _checksum_worker(rank, world, port, q):
    sys.path.insert(0, ROOT)
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    out = []
    try:
        import paper_conf_ipps_leelv14_b200 as av

        torch.cuda.set_device(0)
        assert av.init_distributed(transport="peer", max_report_cap=1 << 12) == "peer"
        reg = synth.C4(1 << 20)
        a, b = rank * reg.n // world, (rank + 1) * reg.n // world
        o, r = reg.slice(a, b - a, device="cuda")
        pinned = torch.empty(24 << 12, dtype=torch.uint8, pin_memory=True).numpy().view(av.REPORT_DTYPE)
        for it in range(6):
            g = av.compare(o, r, reg.abs_tol, reg.rel_tol, 100, report=pinned if it % 2 else None)
            out.append(("cmp", it, g.n, g.n_mismatch, _bits(g.max_abs_err), _bits(g.max_rel_err), g.n_reported,
                        np.array(g.report[: g.n_reported]).tobytes()))
            # the N4 screen between two sharded compares (it used to clobber the
            # exchange's finished-block counter: every later compare returned the
            # previous call's summary with ARC_OK)
            out.append(("sum", it, av.checksum(o), av.checksum(r)))
        av.finalize()
        q.put((rank, out, None))
    except Exception:  # pragma: no cover
        import traceback

        q.put((rank, out, traceback.format_exc()))
    finally:
        dist.destroy_process_group()


@pytest.mark.timeout(600)
@pytest.mark.parametrize("fused", ["1", "0"])
def test_checksum_between_sharded_compares(fused, monkeypatch):
    """compare -> checksum -> compare x 6 on a world-2 peer group: every compare is
    bit-exact against the unsharded oracle on every rank, every checksum equals the
    oracle's checksum of the rank's shard."""
    import oracle

    oracle.build()
    monkeypatch.setenv("ARCV_FUSED_EXCHANGE", fused)
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_checksum_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = {}
    for _ in range(world):
        rank, out, err = q.get(timeout=540)
        assert err is None, f"rank {rank}:\n{err}"
        res[rank] = out
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    reg = synth.C4(1 << 20)
    o, r = reg.slice()
    e = oracle.compare(o.numpy(), r.numpy(), "f64", reg.abs_tol, reg.rel_tol, 100)
    want = (e.n, e.n_mismatch, _bits(e.max_abs_err), _bits(e.max_rel_err), e.n_reported,
            np.ascontiguousarray(e.report).tobytes())
    for rank in range(world):
        a, b = rank * reg.n // world, (rank + 1) * reg.n // world
        sums = (oracle.checksum(o[a:b].numpy()), oracle.checksum(r[a:b].numpy()))
        cmps = [x for x in res[rank] if x[0] == "cmp"]
        assert len(cmps) == 6
        for x in cmps:
            assert x[2:] == want, (rank, x[1], x[2:7], want[:5])
        for x in res[rank]:
            if x[0] == "sum":
                assert (x[2], x[3]) == sums, (rank, x[1])


def _clean_worker(rank, world, port, q):
    sys.path.insert(0, ROOT)
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    out = []
    try:
        import paper_conf_ipps_leelv14_b200 as av

        torch.cuda.set_device(0)
        assert av.init_distributed(transport="peer", max_report_cap=1 << 12) == "peer"
        reg = synth.C2("A")  # clean everywhere: every rank takes the no-report shortcut
        n = 1 << 22
        a, b = rank * n // world, (rank + 1) * n // world
        o, r = reg.slice(a, b - a, device="cuda")
        dirty = synth.C4(1 << 20)  # rank 0 dirty, the others clean
        if rank == 0:
            od, rd = dirty.slice(device="cuda")
        else:
            od, rd = dirty.slice(0, 1 << 18, device="cuda")
            od = rd.clone()
        for it in range(4):
            g = av.compare(o, r, reg.abs_tol, reg.rel_tol, 100)
            out.append(("clean", it, g.n, g.n_mismatch, _bits(g.max_abs_err), _bits(g.max_rel_err), g.n_reported))
            g = av.compare(od, rd, dirty.abs_tol, dirty.rel_tol, 100)
            out.append(("mixed", it, g.n, g.n_mismatch, g.n_reported,
                        tuple(int(i) for i in np.asarray(g.report["index"][: g.n_reported]))))
        av.finalize()
        q.put((rank, out, None))
    except Exception:  # pragma: no cover
        import traceback

        q.put((rank, out, traceback.format_exc()))
    finally:
        dist.destroy_process_group()


@pytest.mark.timeout(600)
@pytest.mark.parametrize("fused", ["1", "0"])
def test_clean_shards_shortcut(fused, monkeypatch):
    """Shards without a single mismatch skip the report phase (the last CTA at the grid
    barrier publishes, the others only keep their counter contract) and still run the
    exchange: all-clean calls and calls where only rank 0 has mismatches, alternating,
    equal to the unsharded oracle / the generator's closed form on every rank."""
    import oracle

    oracle.build()
    monkeypatch.setenv("ARCV_FUSED_EXCHANGE", fused)
    world = 3
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_clean_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = {}
    for _ in range(world):
        rank, out, err = q.get(timeout=540)
        assert err is None, f"rank {rank}:\n{err}"
        res[rank] = out
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    for r in range(1, world):
        assert res[r] == res[0]
    reg = synth.C2("A")
    o, r = reg.slice(0, 1 << 22)
    e = oracle.compare(o.numpy(), r.numpy(), "f32", reg.abs_tol, reg.rel_tol, 100)
    dirty = synth.C4(1 << 20)
    planted = dirty.planted()
    for x in res[0]:
        if x[0] == "clean":
            assert x[2:] == (e.n, e.n_mismatch, _bits(e.max_abs_err), _bits(e.max_rel_err), e.n_reported)
            assert e.n_mismatch == 0
        else:
            assert x[2] == (1 << 20) + 2 * (1 << 18) and x[3] == len(planted)
            assert list(x[5]) == planted[:100]
