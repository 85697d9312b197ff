#!/usr/bin/env python
"""Benchmark: verified GB/s (both arrays read) of the kernel-verification comparison.

Workload (BASELINE.json configs[3], the config the metric's "1/2/4/8 B200" is
quoted on): C4 -- fp64, 2^29 elements per array (4 GiB each, 8 GiB read per
step), 512 injected mismatches + 4 NaN/number pairs, abs_tol 1e-6, rel_tol
1e-5, max_report 2^20.  At N GPUs the array is split into N contiguous shards
(one per rank, generated on that rank) and every step is one collective
arc_verify_compare (local kernel + NCCL merge): strong scaling, fixed total.

One step = one arc_verify_compare call on HBM-resident arrays (the whole hot
path: stream + predicate + reductions + ordered compaction + summary/report to
the host).  value = global bytes (2 * n * 8) * K / max-over-ranks device time.
e2e = the same metric through the same C-ABI call with the arrays in pinned
HOST memory: the library streams them to the GPU in chunks overlapped with the
comparison, so H2D copies are inside the timed region.

  python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

N_C4 = 1 << 29
ES = 8


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=200)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--n", "--n-elements", dest="n", type=int, default=N_C4,
                    help="elements per array (default: C4's 2^29); --n-elements under torchrun")
    ap.add_argument("--e2e-steps", type=int, default=5)
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-configs", action="store_true", help="skip the other BASELINE configs (N = 1)")
    ap.add_argument("--profile", action="store_true", help="short run for ncu (no clocks/e2e/cpu)")
    return ap.parse_args()


def measured_peak():
    path = os.path.join(ROOT, "MEASURED_PEAKS.json")
    try:
        with open(path) as f:
            return float(json.load(f)["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs, copy r+w)"
    except Exception:
        return 6650.0, "fallback (B200_PROFILING.md)"


def ncu_traffic():
    """dram bytes (read+write) per launch of the compare kernel from the committed ncu capture."""
    path = os.path.join(ROOT, "profiles", "ncu_summary.json")
    try:
        with open(path) as f:
            d = json.load(f)
        return d.get("c4_dram_bytes_per_launch")
    except Exception:
        return None


class ClockSampler:
    """Samples SM clock and throttle reasons via NVML while the timed region runs."""

    REASONS = {
        0x1: "gpu_idle", 0x2: "applications_clocks_setting", 0x4: "sw_power_cap", 0x8: "hw_slowdown",
        0x10: "sync_boost", 0x20: "sw_thermal_slowdown", 0x40: "hw_thermal_slowdown",
        0x80: "hw_power_brake_slowdown", 0x100: "display_clock_setting",
    }

    def __init__(self, device: int):
        self.samples, self.reasons, self.ok = [], set(), False
        self.max_mhz = None
        try:
            import pynvml

            pynvml.nvmlInit()
            self.nv = pynvml
            self.h = pynvml.nvmlDeviceGetHandleByIndex(device)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
            self.ok = True
        except Exception as e:  # pragma: no cover
            self.err = str(e)
        self._stop = threading.Event()
        self.interval = 0.005  # seconds between NVML samples

    def _run(self):
        while not self._stop.is_set():
            try:
                self.samples.append(self.nv.nvmlDeviceGetClockInfo(self.h, self.nv.NVML_CLOCK_SM))
                fn = getattr(self.nv, "nvmlDeviceGetCurrentClocksEventReasons", None) or \
                    self.nv.nvmlDeviceGetCurrentClocksThrottleReasons
                mask = fn(self.h)
                for bit, name in self.REASONS.items():
                    if mask & bit and bit != 0x1:
                        self.reasons.add(name)
            except Exception:
                pass
            time.sleep(self.interval)

    def __enter__(self):
        if self.ok:
            self.t = threading.Thread(target=self._run, daemon=True)
            self.t.start()
        return self

    def __exit__(self, *a):
        if self.ok:
            self._stop.set()
            self.t.join()

    def summary(self):
        if not self.ok or not self.samples:
            return {"sm_mhz": None, "sm_max_mhz": self.max_mhz, "reasons": ["unavailable"], "samples": 0}
        return {"sm_mhz": statistics.median(self.samples), "sm_max_mhz": self.max_mhz,
                "reasons": sorted(self.reasons), "samples": len(self.samples)}


# ---------------------------------------------------------------- reference
def _host_cores() -> int:
    return len(os.sched_getaffinity(0))


def host_description() -> dict:
    """lscpu model / sockets / cores of the host the oracle ran on."""
    import subprocess

    d = {"affinity_threads": _host_cores()}
    try:
        out = subprocess.run(["lscpu"], capture_output=True, text=True, timeout=10).stdout
        keys = {"Model name": "model", "Socket(s)": "sockets", "Core(s) per socket": "cores_per_socket",
                "Thread(s) per core": "threads_per_core", "CPU(s)": "cpus", "L3 cache": "l3",
                "Hypervisor vendor": "hypervisor"}
        for line in out.splitlines():
            k, _, v = line.partition(":")
            if k.strip() in keys:
                d[keys[k.strip()]] = v.strip()
    except Exception as e:  # pragma: no cover
        d["lscpu_error"] = str(e)
    return d


def run_reference(args, rank):
    """The oracle, as it stands, on all host cores (contiguous chunks in host
    threads, merged by the oracle's own merge_shards): each step a bounded
    sample of C4 (its first 2^24 elements)."""
    if rank != 0:
        return
    from concurrent.futures import ThreadPoolExecutor

    import oracle
    import synth

    oracle.build()
    sample = min(1 << 24, args.n)
    c4 = synth.C4(args.n)
    out, ref = c4.slice(0, sample)
    o, r = out.numpy(), ref.numpy()
    cores = _host_cores()
    with ThreadPoolExecutor(cores) as pool:
        def step():
            return oracle.compare_threads(o, r, "f64", c4.abs_tol, c4.rel_tol, c4.max_report, cores, pool)
        for _ in range(args.warmup):
            res = step()
        t0 = time.perf_counter()
        for _ in range(args.steps):
            res = step()
        dt = time.perf_counter() - t0
    planted = [i for i in c4.planted() if i < sample]
    gbs = 2 * o.size * ES * args.steps / dt / 1e9
    line = {
        "impl": "reference", "metric": "verified GB/s (both arrays read)", "value": round(gbs, 3),
        "unit": "GB/s", "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup,
        "ms_per_step": round(dt / args.steps * 1e3, 3), "higher_is_better": True, "scaling": "strong",
        "vs_baseline": None, "dtype": "f64", "data": "synthetic",
        "config": {"workload": f"C4 sample: first {o.size} elements (fp64) of the C4 arrays per step",
                   "parallelism": f"{cores} host threads (oracle on contiguous chunks + merge_shards)"},
        "parity": "ok" if list(res.report["index"]) == planted[: c4.max_report] else "FAIL",
        "cpu_baseline": {"value": round(gbs, 3), "unit": "GB/s", "cores": cores, "kind": "oracle",
                         "sample": f"first 2^24 of 2^29 C4 elements, {args.steps} steps",
                         "host": host_description()},
        "e2e": {"value": round(gbs, 3), "unit": "GB/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)


def cpu_baseline(c4, out_dev, ref_dev):
    """The oracle timed on the host over bounded samples of the same C4 arrays:
    on all host cores (primary: first 2^26 elements, contiguous chunks in host
    threads + merge_shards) and on one core (first 2^24 elements)."""
    from concurrent.futures import ThreadPoolExecutor

    import oracle

    oracle.build()
    cores = _host_cores()
    big = min(1 << 26, out_dev.numel())
    o, r = out_dev[:big].cpu().numpy(), ref_dev[:big].cpu().numpy()

    def timed(fn, budget=5.0, max_reps=20):
        reps, t_total = 0, 0.0
        while t_total < budget and reps < max_reps:
            t0 = time.perf_counter()
            fn()
            t_total += time.perf_counter() - t0
            reps += 1
        return reps, t_total

    with ThreadPoolExecutor(cores) as pool:
        reps, t_all = timed(lambda: oracle.compare_threads(o, r, "f64", c4.abs_tol, c4.rel_tol, c4.max_report,
                                                           cores, pool))
    gbs_all = 2 * big * ES * reps / t_all / 1e9
    small = min(1 << 24, big)
    reps1, t_one = timed(lambda: oracle.compare(o[:small], r[:small], "f64", c4.abs_tol, c4.rel_tol, c4.max_report))
    gbs_one = 2 * small * ES * reps1 / t_one / 1e9
    return {"value": round(gbs_all, 3), "unit": "GB/s", "cores": cores, "kind": "oracle",
            "host": host_description(),
            "sample": f"first 2^26 of the 2^29 C4 elements (fp64) on {cores} host threads (oracle on "
                      f"contiguous chunks + merge_shards), {reps} repetition(s), {t_all:.1f} s",
            "single_core": {"value": round(gbs_one, 3), "unit": "GB/s", "cores": 1,
                            "sample": f"first 2^24 C4 elements, {reps1} repetition(s), {t_one:.1f} s"}}


def other_configs(av, synth, stream, steps=10):
    """Per-call device time of the other BASELINE configs at N = 1 (C1, C2 A/B, C3 as one
    batched call, C5), each checked against its generator's closed form.  Arrays smaller than
    4x L2 get an L2 flush between calls (outside the timed events)."""
    import torch

    L2 = torch.cuda.get_device_properties(0).L2_cache_size
    scratch = torch.empty(2 * L2, dtype=torch.uint8, device="cuda")
    rep = torch.empty(24 * (1 << 20), dtype=torch.uint8, pin_memory=True).numpy().view(av.REPORT_DTYPE)
    out = {}

    def timed(fn, nbytes, flush):
        for _ in range(3):
            res = fn()
        tot = 0.0
        for _ in range(steps):
            if flush:
                scratch.fill_(1)
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            res = fn()
            e1.record(stream)
            torch.cuda.synchronize()
            tot += e0.elapsed_time(e1)
        us = 1e3 * tot / steps
        return res, {"per_call_us": round(us, 1), "gbs": round(nbytes / us / 1e3, 1), "l2_flush": flush}

    def idx(r):
        return [int(i) for i in r.report["index"]]

    c1 = synth.C1()
    o, r = c1.slice(device="cuda")
    res, d = timed(av.prepare(o, r, c1.abs_tol, c1.rel_tol, c1.max_report, report=rep), 2 * o.numel() * 4, True)
    d["parity"] = "ok" if idx(res) == c1.planted() else "FAIL"
    out["C1 fp32 2^20"] = d
    del o, r
    for v in ("A", "B"):
        c2 = synth.C2(v)
        o, r = c2.slice(device="cuda")
        res, d = timed(av.prepare(o, r, c2.abs_tol, c2.rel_tol, c2.max_report, report=rep), 2 * o.numel() * 4,
                       False)
        d["parity"] = "ok" if idx(res) == c2.planted() else "FAIL"
        out[f"C2{v} Jacobi-2D fp32 8192^2"] = d
        del o, r
    regs = synth.c3_regions()
    data = [rg.slice(device="cuda") for rg in regs]
    nb = sum(2 * o.numel() * o.element_size() for o, _ in data)
    pb = av.prepare_batch([(o, r, rg.abs_tol, rg.rel_tol, rg.max_report, rg.name) for rg, (o, r) in zip(regs, data)])
    res, d = timed(pb, nb, True)
    d["parity"] = "ok" if all(idx(x) == rg.planted()[: rg.max_report] for x, rg in zip(res, regs)) else "FAIL"
    out["C3 twelve regions, one batched call"] = d
    del data, pb
    c5 = synth.C5()
    o, r = c5.slice(device="cuda")
    drep = torch.empty(24 * c5.max_report, dtype=torch.uint8, device="cuda")
    res, d = timed(av.prepare(o, r, 0, 0, c5.max_report, report=drep), 2 * o.numel() * 4, False)
    first = drep[: 24 * 8].cpu().numpy().view(av.REPORT_DTYPE)
    d["parity"] = "ok" if (res.n_mismatch == c5.n // 2 and res.n_reported == c5.max_report and
                           [int(i) for i in first["index"]] == list(range(1, 17, 2))) else "FAIL"
    d["report"] = "device buffer (2^20 entries)"
    out["C5 int32 2^30, 50% mismatches"] = d
    del o, r, drep, scratch
    torch.cuda.empty_cache()
    return out


# --------------------------------------------------------------------- ours
def main():
    args = parse()
    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local_rank = int(os.environ.get("LOCAL_RANK", "0"))
    if args.impl == "reference":
        return run_reference(args, rank)

    import torch
    import torch.distributed as dist

    import paper_conf_ipps_leelv14_b200 as av
    import synth

    assert world == args.gpus, f"--gpus {args.gpus} but WORLD_SIZE {world}"
    # ARCV_BENCH_ONE_GPU=1 (diagnostic, tests only): every rank on cuda:0, gloo for
    # the host-side collectives, peer windows between the processes -- exercises
    # the N > 1 code path on a one-GPU box (its numbers mean nothing)
    one_gpu = os.environ.get("ARCV_BENCH_ONE_GPU") == "1"
    dev = 0 if one_gpu else local_rank
    torch.cuda.set_device(dev)
    exchange = None
    if world > 1:
        if one_gpu:
            dist.init_process_group("gloo")
        else:
            dist.init_process_group("nccl", device_id=torch.device("cuda", local_rank))
        # the device-driven peer-memory exchange (CUDA IPC windows over NVLink);
        # NCCL only as the fallback when the windows cannot be mapped
        exchange = av.init_distributed(transport="peer" if one_gpu else "auto", max_report_cap=1 << 20)
    else:
        av.init(dev)
    red_dev = "cpu" if one_gpu else "cuda"

    n = args.n
    lo, hi = rank * n // world, (rank + 1) * n // world
    c4 = synth.C4(n)
    out, ref = c4.slice(lo, hi - lo, device="cuda")
    torch.cuda.synchronize()
    mr = c4.max_report
    # caller-owned report buffer, allocated once (pinned host memory, numpy view)
    report = torch.empty(24 * mr, dtype=torch.uint8, pin_memory=True).numpy().view(av.REPORT_DTYPE)

    # the public prepared-call API: arguments validated/marshalled once, each step
    # is one arc_verify_compare through the C ABI
    step = av.prepare(out, ref, c4.abs_tol, c4.rel_tol, mr, report=report)

    def barrier():
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()

    for _ in range(args.warmup):
        res = step()
    barrier()
    # Kernel time for the roofline: the library's CUDA events around every K1
    # launch (on the stream it launches on), over K steps of the same call.
    # Those two cudaEventRecord per launch cost ~2.7 us of host time per call on
    # these boxes (1.6 % of a 2^26-element p = 8 shard step, profiles/
    # r02am_timing.log), so they run in their own pass of K steps right before
    # the timed pass, which carries no per-launch events.
    av.arc_verify_set_timing(True)
    av.arc_verify_kernel_stats(reset=True)
    for _ in range(args.steps):
        res = step()
    torch.cuda.synchronize()
    launches, kern_ms = av.arc_verify_kernel_stats(reset=True)
    av.arc_verify_set_timing(False)
    barrier()
    launches0 = av.arc_verify_launch_count()
    stream = torch.cuda.current_stream()
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    sampler = ClockSampler(dev) if not args.profile else None
    barrier()
    if sampler:
        sampler.__enter__()
    ev0.record(stream)
    for _ in range(args.steps):
        res = step()
    ev1.record(stream)
    torch.cuda.synchronize()
    if sampler:
        sampler.__exit__()
    ms = ev0.elapsed_time(ev1)
    gpu_launches = av.arc_verify_launch_count() - launches0
    t = torch.tensor([ms, kern_ms / max(launches, 1)], dtype=torch.float64, device=red_dev)
    if world > 1:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    ms_max, kern_avg_ms = float(t[0]), float(t[1])

    # in-run read-only ceiling: the same bulk-copy pipeline with the predicate off
    probe = None
    if not args.profile:
        probe = av.arc_verify_probe_read(out.data_ptr(), ref.data_ptr(), (hi - lo) * ES, iters=10)

    # parity of the timed result against the generator's closed form
    planted = c4.planted()
    parity = (res.n_mismatch == len(planted) and list(res.report["index"]) == planted)

    total_bytes = 2 * n * ES
    value = total_bytes * args.steps / (ms_max / 1e3) / 1e9
    local_bytes = 2 * (hi - lo) * ES
    achieved = local_bytes / (kern_avg_ms / 1e3) / 1e9
    peak, peak_src = measured_peak()

    # ------------------------------------------------------------------ e2e
    e2e = None
    if not args.no_e2e and not args.profile:
        ho = out.cpu().pin_memory()
        hr = ref.cpu().pin_memory()
        del_out = None
        step_h = av.prepare(ho, hr, c4.abs_tol, c4.rel_tol, mr, report=report)
        step_h()
        barrier()
        t0 = torch.cuda.Event(enable_timing=True)
        t1 = torch.cuda.Event(enable_timing=True)
        t0.record(stream)
        for _ in range(args.e2e_steps):
            rh = step_h()
        t1.record(stream)
        torch.cuda.synchronize()
        te = torch.tensor([t0.elapsed_time(t1)], dtype=torch.float64, device=red_dev)
        if world > 1:
            dist.all_reduce(te, op=dist.ReduceOp.MAX)
        e2e_ms = float(te[0])
        parity = parity and rh.n_mismatch == res.n_mismatch
        e2e = {"value": round(total_bytes * args.e2e_steps / (e2e_ms / 1e3) / 1e9, 3), "unit": "GB/s",
               "h2d_bytes_per_step": 2 * (hi - lo) * ES * world,
               "d2h_bytes_per_step": (32 + 24 * rh.n_reported) * world,
               "steps": args.e2e_steps, "ms_per_step": round(e2e_ms / args.e2e_steps, 3),
               "path": "arc_verify_compare with pinned host out/ref (chunked H2D overlapped with compare)"}
        # the paper's own data flow: the kernel output is already in HBM,
        # the sequential reference lives in host memory -> half the PCIe bytes
        step_r = av.prepare(out, hr, c4.abs_tol, c4.rel_tol, mr, report=report)
        step_r()
        barrier()
        t0.record(stream)
        for _ in range(args.e2e_steps):
            rr = step_r()
        t1.record(stream)
        torch.cuda.synchronize()
        te = torch.tensor([t0.elapsed_time(t1)], dtype=torch.float64, device=red_dev)
        if world > 1:
            dist.all_reduce(te, op=dist.ReduceOp.MAX)
        parity = parity and rr.n_mismatch == res.n_mismatch
        e2e["ref_on_host"] = {
            "value": round(total_bytes * args.e2e_steps / (float(te[0]) / 1e3) / 1e9, 3), "unit": "GB/s",
            "h2d_bytes_per_step": (hi - lo) * ES * world, "d2h_bytes_per_step": (32 + 24 * rr.n_reported) * world,
            "path": "out in HBM, ref in pinned host memory (the paper's data flow, P:171)"}
        del ho, hr, del_out

    if rank == 0:
        line = {
            "metric": "verified GB/s (both arrays read)",
            "value": round(value, 3), "unit": "GB/s", "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": round(ms_max / args.steps, 4), "higher_is_better": True,
            "scaling": "strong", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": {"workload": "C4: fp64 2^29 elements per array (4 GiB each), 512 injected + 4 NaN "
                                   "pairs, abs_tol 1e-6, rel_tol 1e-5, max_report 2^20",
                       "n": n, "parallelism": f"shard{world}" if world > 1 else "single",
                       "exchange": exchange,
                       "l2": "inputs (8 GiB) larger than L2 (126 MB); no flush",
                       "report": "caller-owned pinned host buffer (2^20 entries)"},
            "parity": "ok" if parity else "FAIL",
            "gpu_launches": int(gpu_launches),
            "roofline": {"bound": "hbm", "achieved": round(achieved, 1), "peak": peak, "unit": "GB/s",
                         "frac": round(achieved / peak, 4),
                         # the committed ncu capture is of this exact launch only at N = 1 on C4
                         "traffic": ncu_traffic() if (world == 1 and n == N_C4) else None,
                         "traffic_source": ("committed ncu --set full capture of this launch "
                                            "(profiles/ncu_summary.json: dram__bytes_read.sum + "
                                            "dram__bytes_write.sum), not measured in this run"
                                            if (world == 1 and n == N_C4) else None),
                         "kernel": "arcv_stream_kernel (report phase fused in its tail)", "kernel_ms_avg": round(kern_avg_ms, 4),
                         "kernel_ms_source": ("CUDA events around each K1 launch on its stream (library timing), "
                                              f"{launches} launches in a pass of the same {args.steps} steps just "
                                              "before the timed pass (per-launch events stay out of `value`)"),
                         "algorithmic_bytes_per_launch": local_bytes, "peak_source": peak_src,
                         "read_probe_gbs": round(probe, 1) if probe else None,
                         "frac_of_read_probe": round(achieved / probe, 4) if probe else None},
            "e2e": e2e,
        }
        if sampler:
            line["clocks"] = sampler.summary()
        if world == 1 and not args.no_cpu_baseline and not args.profile:
            line["cpu_baseline"] = cpu_baseline(c4, out, ref)
        if world == 1 and not args.no_configs and not args.profile and n == N_C4:
            del out, ref
            torch.cuda.empty_cache()
            line["other_configs"] = other_configs(av, synth, stream)
        print(json.dumps(line), flush=True)
    av.finalize()
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
