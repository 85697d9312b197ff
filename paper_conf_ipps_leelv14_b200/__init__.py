"""paper_conf_ipps_leelv14_b200 -- B200-native kernel-verification result comparison.

Thin ctypes binding over ``libarcverify.so`` (C ABI: include/arc_verify.h).
The functions named ``arc_verify_*`` mirror the C entry points one to one and
only marshal arguments; every step of the comparison runs in the library's
CUDA kernels.  ``compare`` / ``batch`` are conveniences over torch tensors
(PyTorch is used for device memory, streams and process groups only).

There is no CPU fallback: importing this package without the built library
raises ImportError.  Build it with ``python paper_conf_ipps_leelv14_b200/_build.py``
or ``__graft_entry__.build()``.

Paper: S. Lee, D. Li, J. S. Vetter, "Interactive Program Debugging and
Optimization for Directive-Based, Efficient GPU Computing", IPDPS 2014,
sec. III-A: verify each GPU kernel's outputs against the
sequential CPU outputs under a user-configurable error margin and report the
differences.
"""
from __future__ import annotations

import ctypes
import os
from dataclasses import dataclass, field
from typing import Optional, Sequence

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("ARCV_LIB_PATH") or os.path.join(_HERE, "libarcverify.so")  # override: diagnostics

ARC_OK, ARC_E_INVAL, ARC_E_NOINIT, ARC_E_CUDA, ARC_E_NCCL, ARC_E_NOMEM, ARC_E_UNSUPPORTED = 0, -1, -2, -3, -4, -5, -6
ARC_F32, ARC_F64, ARC_I32, ARC_I64, ARC_U8 = 0, 1, 2, 3, 4
DTYPE_CODES = {"f32": ARC_F32, "f64": ARC_F64, "i32": ARC_I32, "i64": ARC_I64, "u8": ARC_U8}

EXPORTED = [
    "arc_verify_init", "arc_verify_compare", "arc_verify_batch", "arc_verify_finalize",
    "arc_verify_strerror", "arc_verify_last_error", "arc_verify_set_stream",
    "arc_verify_get_unique_id", "arc_verify_set_timing", "arc_verify_kernel_stats",
    "arc_verify_version", "arc_verify_merge_plan", "arc_verify_packet_bytes",
    "arc_verify_shard_local", "arc_verify_shard_merge", "arc_verify_probe_read", "arc_verify_compare_ex",
    "arc_verify_checksum", "arc_verify_selected", "arc_verify_batch_selected", "arc_verify_format_result",
    "arc_verify_peer_export", "arc_verify_peer_open", "arc_verify_launch_count", "arc_verify_build_info",
    "arc_verify_peer_stats",
]


class arc_mismatch_t(ctypes.Structure):
    _fields_ = [("index", ctypes.c_uint64), ("out_bits", ctypes.c_uint64), ("ref_bits", ctypes.c_uint64)]


class arc_verify_result_t(ctypes.Structure):
    _fields_ = [
        ("n", ctypes.c_uint64), ("n_mismatch", ctypes.c_uint64),
        ("max_abs_err", ctypes.c_double), ("max_rel_err", ctypes.c_double),
        ("n_reported", ctypes.c_uint64), ("report", ctypes.c_void_p),
    ]


class arc_verify_opts_t(ctypes.Structure):
    _fields_ = [("device", ctypes.c_int), ("stream", ctypes.c_void_p), ("rank", ctypes.c_int),
                ("nranks", ctypes.c_int), ("nccl_unique_id", ctypes.c_void_p)]


ARC_CHECK_MIN_VALUE, ARC_CHECK_VALUE_BOUNDS = 1, 2


class arc_verify_check_t(ctypes.Structure):
    _fields_ = [("flags", ctypes.c_uint32), ("min_value", ctypes.c_double), ("lo", ctypes.c_double),
                ("hi", ctypes.c_double)]


class arc_verify_region_t(ctypes.Structure):
    _fields_ = [("out", ctypes.c_void_p), ("ref", ctypes.c_void_p), ("n", ctypes.c_uint64),
                ("dtype", ctypes.c_int), ("abs_tol", ctypes.c_double), ("rel_tol", ctypes.c_double),
                ("max_report", ctypes.c_uint64), ("name", ctypes.c_char_p),
                ("check", ctypes.POINTER(arc_verify_check_t))]


class arc_shard_header_t(ctypes.Structure):
    _fields_ = [("n", ctypes.c_uint64), ("n_mismatch", ctypes.c_uint64),
                ("max_abs_bits", ctypes.c_uint64), ("max_rel_bits", ctypes.c_uint64)]


class arc_shard_plan_t(ctypes.Structure):
    _fields_ = [("index_offset", ctypes.c_uint64), ("prefix", ctypes.c_uint64), ("contrib", ctypes.c_uint64)]


CUDA_STREAM_LEGACY = 1  # cudaStreamLegacy

REPORT_DTYPE = np.dtype([("index", "<u8"), ("out_bits", "<u8"), ("ref_bits", "<u8")])


def _load() -> ctypes.CDLL:
    if not os.path.exists(LIB_PATH):
        raise ImportError(f"{LIB_PATH} is missing: build it with __graft_entry__.build() "
                          "(there is no CPU fallback)")
    lib = ctypes.CDLL(LIB_PATH)
    P, U64, I, D, SZ = ctypes.c_void_p, ctypes.c_uint64, ctypes.c_int, ctypes.c_double, ctypes.c_size_t
    sig = {
        "arc_verify_init": (I, [ctypes.POINTER(arc_verify_opts_t)]),
        "arc_verify_compare": (I, [P, P, U64, I, D, D, U64, ctypes.POINTER(arc_verify_result_t)]),
        "arc_verify_batch": (I, [ctypes.POINTER(arc_verify_region_t), SZ, ctypes.POINTER(arc_verify_result_t)]),
        "arc_verify_finalize": (I, []),
        "arc_verify_strerror": (ctypes.c_char_p, [I]),
        "arc_verify_last_error": (ctypes.c_char_p, []),
        "arc_verify_set_stream": (I, [P]),
        "arc_verify_get_unique_id": (I, [P]),
        "arc_verify_set_timing": (I, [I]),
        "arc_verify_kernel_stats": (I, [ctypes.POINTER(U64), ctypes.POINTER(D), I]),
        "arc_verify_version": (ctypes.c_uint32, []),
        "arc_verify_build_info": (ctypes.c_char_p, []),
        "arc_verify_peer_stats": (I, [ctypes.POINTER(U64), I]),
        "arc_verify_merge_plan": (I, [ctypes.POINTER(arc_shard_header_t), I, U64,
                                      ctypes.POINTER(arc_shard_plan_t), ctypes.POINTER(arc_shard_header_t)]),
        "arc_verify_packet_bytes": (SZ, [U64]),
        "arc_verify_shard_local": (I, [P, P, U64, I, D, D, U64, P, U64]),
        "arc_verify_shard_merge": (I, [P, I, U64, U64, ctypes.POINTER(arc_verify_result_t)]),
        "arc_verify_probe_read": (I, [P, P, U64, I, ctypes.POINTER(D)]),
        "arc_verify_compare_ex": (I, [P, P, U64, I, D, D, U64, ctypes.POINTER(arc_verify_check_t),
                                      ctypes.POINTER(arc_verify_result_t)]),
        "arc_verify_checksum": (I, [P, U64, ctypes.POINTER(U64)]),
        "arc_verify_selected": (I, [ctypes.c_char_p, ctypes.c_char_p]),
        "arc_verify_batch_selected": (I, [ctypes.POINTER(arc_verify_region_t), SZ, ctypes.c_char_p,
                                          ctypes.POINTER(arc_verify_result_t), P]),
        "arc_verify_format_result": (I, [ctypes.c_char_p, I, D, D, ctypes.POINTER(arc_verify_result_t), U64,
                                         ctypes.c_char_p, SZ]),
        "arc_verify_peer_export": (I, [U64, P]),
        "arc_verify_peer_open": (I, [P]),
        "arc_verify_launch_count": (U64, []),
    }
    for name, (res, args) in sig.items():
        f = getattr(lib, name)
        f.restype, f.argtypes = res, args
    return lib


_lib = _load()


class ArcVerifyError(RuntimeError):
    def __init__(self, status: int, where: str):
        self.status = status
        msg = _lib.arc_verify_strerror(status).decode()
        detail = _lib.arc_verify_last_error().decode()
        super().__init__(f"{where}: {msg} ({status}){': ' + detail if detail else ''}")


def _check(status: int, where: str) -> None:
    if status != ARC_OK:
        raise ArcVerifyError(status, where)


# --------------------------------------------------------- raw C entry points
def arc_verify_init(device: int = 0, stream: Optional[int] = None, rank: int = 0, nranks: int = 1,
                    nccl_unique_id: Optional[bytes] = None) -> None:
    opts = arc_verify_opts_t(device, stream or None, rank, nranks, None)
    buf = None
    if nccl_unique_id is not None:
        buf = ctypes.create_string_buffer(bytes(nccl_unique_id), 128)
        opts.nccl_unique_id = ctypes.cast(buf, ctypes.c_void_p)
    _check(_lib.arc_verify_init(ctypes.byref(opts)), "arc_verify_init")


def arc_verify_finalize() -> None:
    _check(_lib.arc_verify_finalize(), "arc_verify_finalize")


def arc_verify_compare(out_ptr: int, ref_ptr: int, n: int, dtype: int, abs_tol: float, rel_tol: float,
                       max_report: int, result: arc_verify_result_t) -> None:
    _check(_lib.arc_verify_compare(out_ptr or None, ref_ptr or None, n, dtype, abs_tol, rel_tol, max_report,
                                   ctypes.byref(result)), "arc_verify_compare")


def arc_verify_batch(regions, results) -> None:
    n = len(regions)
    _check(_lib.arc_verify_batch(regions, n, results), "arc_verify_batch")


def arc_verify_set_stream(stream: int) -> None:
    _check(_lib.arc_verify_set_stream(stream), "arc_verify_set_stream")


def arc_verify_get_unique_id() -> bytes:
    buf = ctypes.create_string_buffer(128)
    _check(_lib.arc_verify_get_unique_id(buf), "arc_verify_get_unique_id")
    return buf.raw


def arc_verify_set_timing(enable: bool) -> None:
    _check(_lib.arc_verify_set_timing(int(enable)), "arc_verify_set_timing")


def arc_verify_kernel_stats(reset: bool = False) -> tuple[int, float]:
    n, ms = ctypes.c_uint64(), ctypes.c_double()
    _check(_lib.arc_verify_kernel_stats(ctypes.byref(n), ctypes.byref(ms), int(reset)), "arc_verify_kernel_stats")
    return int(n.value), float(ms.value)


def arc_verify_launch_count() -> int:
    """Kernels the library launched since init (every kernel it owns)."""
    return int(_lib.arc_verify_launch_count())


def arc_verify_build_info() -> str:
    return _lib.arc_verify_build_info().decode()


def arc_verify_version() -> int:
    return int(_lib.arc_verify_version())


def arc_verify_packet_bytes(entries: int) -> int:
    return int(_lib.arc_verify_packet_bytes(entries))


def arc_verify_merge_plan(headers: Sequence[tuple], max_report: int):
    """headers: [(n, n_mismatch, max_abs_bits, max_rel_bits)] in rank order (host only)."""
    p = len(headers)
    H = (arc_shard_header_t * p)(*[arc_shard_header_t(*h) for h in headers])
    plan = (arc_shard_plan_t * p)()
    g = arc_shard_header_t()
    _check(_lib.arc_verify_merge_plan(H, p, max_report, plan, ctypes.byref(g)), "arc_verify_merge_plan")
    return ([(x.index_offset, x.prefix, x.contrib) for x in plan],
            (g.n, g.n_mismatch, g.max_abs_bits, g.max_rel_bits))


def arc_verify_shard_local(out_ptr, ref_ptr, n, dtype, abs_tol, rel_tol, max_report, packet_ptr, packet_entries):
    _check(_lib.arc_verify_shard_local(out_ptr or None, ref_ptr or None, n, dtype, abs_tol, rel_tol, max_report,
                                       packet_ptr, packet_entries), "arc_verify_shard_local")


def arc_verify_shard_merge(gathered_ptr, nranks, packet_entries, max_report, result: arc_verify_result_t):
    _check(_lib.arc_verify_shard_merge(gathered_ptr, nranks, packet_entries, max_report, ctypes.byref(result)),
           "arc_verify_shard_merge")


def arc_verify_peer_export(max_report_cap: int) -> bytes:
    """Allocate this rank's exchange window; returns its 64-byte IPC handle."""
    buf = ctypes.create_string_buffer(64)
    _check(_lib.arc_verify_peer_export(max_report_cap, buf), "arc_verify_peer_export")
    return buf.raw


def arc_verify_peer_stats(reset: bool = False) -> tuple[int, int]:
    """(bytes pulled from owners' packets, bytes read from a forwarding neighbour)."""
    b = (ctypes.c_uint64 * 2)()
    _check(_lib.arc_verify_peer_stats(b, int(reset)), "arc_verify_peer_stats")
    return int(b[0]), int(b[1])


def arc_verify_peer_open(handles: Sequence[bytes]) -> None:
    """Map every rank's window (handles in rank order) and enable the peer path."""
    blob = b"".join(bytes(h) for h in handles)
    buf = ctypes.create_string_buffer(blob, len(blob))
    _check(_lib.arc_verify_peer_open(buf), "arc_verify_peer_open")


def arc_verify_probe_read(a_ptr: int, b_ptr: int, nbytes: int, iters: int = 10) -> float:
    """Diagnostic: read-only streaming GB/s of the comparison's pipeline (no predicate)."""
    g = ctypes.c_double()
    _check(_lib.arc_verify_probe_read(a_ptr, b_ptr, nbytes, iters, ctypes.byref(g)), "arc_verify_probe_read")
    return float(g.value)


def arc_verify_checksum(ptr: int, nbytes: int) -> tuple[int, int]:
    out = (ctypes.c_uint64 * 2)()
    _check(_lib.arc_verify_checksum(ptr or None, nbytes, out), "arc_verify_checksum")
    return int(out[0]), int(out[1])


def checksum(t) -> tuple[int, int]:
    """Debug-assertion checksum (sum, xor) of a CUDA tensor's bytes (N4)."""
    if not t.is_contiguous():
        raise ValueError("tensor must be contiguous")
    nb = t.numel() * t.element_size()
    return arc_verify_checksum(t.data_ptr() if nb else 0, nb)


def arc_verify_selected(options: Optional[str], name: str) -> bool:
    st = _lib.arc_verify_selected(options.encode() if options is not None else None, name.encode())
    if st < 0:
        raise ArcVerifyError(st, "arc_verify_selected")
    return bool(st)


def arc_verify_format_result(name: str, dtype: int, abs_tol: float, rel_tol: float, result: arc_verify_result_t,
                             max_entries: int = 10) -> str:
    cap = 4096 + 256 * max_entries
    buf = ctypes.create_string_buffer(cap)
    st = _lib.arc_verify_format_result(name.encode() if name else None, dtype, abs_tol, rel_tol,
                                       ctypes.byref(result), max_entries, buf, cap)
    if st < 0:
        raise ArcVerifyError(st, "arc_verify_format_result")
    return buf.value.decode()


def format_result(name: str, dtype: str, abs_tol: float, rel_tol: float, res: "Result",
                  max_entries: int = 10) -> str:
    """Report text for a Result (host numpy report) -- P:199 "reported to the user"."""
    r = arc_verify_result_t(res.n, res.n_mismatch, res.max_abs_err, res.max_rel_err, res.n_reported, None)
    rep = np.ascontiguousarray(res.report, dtype=REPORT_DTYPE) if res.n_reported else None
    if rep is not None:
        r.report = rep.ctypes.data
    return arc_verify_format_result(name, DTYPE_CODES[dtype], abs_tol, rel_tol, r, max_entries)


# ------------------------------------------------------------- conveniences
@dataclass
class Result:
    n: int
    n_mismatch: int
    max_abs_err: float
    max_rel_err: float
    n_reported: int
    report: np.ndarray = field(repr=False)  # REPORT_DTYPE (host), or a device tensor view


_TORCH_CODES = None


def dtype_code(t) -> int:
    global _TORCH_CODES
    import torch

    if _TORCH_CODES is None:
        _TORCH_CODES = {torch.float32: ARC_F32, torch.float64: ARC_F64, torch.int32: ARC_I32,
                        torch.int64: ARC_I64, torch.uint8: ARC_U8}
    try:
        return _TORCH_CODES[t.dtype]
    except KeyError:
        raise TypeError(f"unsupported dtype {t.dtype}") from None


_state = {"init": False, "nranks": 1}


def init(device: Optional[int] = None, stream=None, rank: int = 0, nranks: int = 1,
         nccl_unique_id: Optional[bytes] = None) -> None:
    """Initialise on ``device`` enqueuing on ``stream`` (default: torch's current stream)."""
    import torch

    if device is None:
        device = torch.cuda.current_device()
    if stream is None:
        stream = torch.cuda.current_stream(device)
    handle = stream.cuda_stream if hasattr(stream, "cuda_stream") else stream
    if not handle:
        handle = CUDA_STREAM_LEGACY  # torch's default stream is the legacy NULL stream
    arc_verify_init(device, handle, rank, nranks, nccl_unique_id)
    _state["init"] = True
    _state["nranks"] = nranks


def init_distributed(group=None, transport: str = "peer", max_report_cap: int = 1 << 20) -> str:
    """Sharded init over a torch.distributed group (any backend; only small host
    objects travel through it).  Returns the exchange in use.

    transport="peer": peer-memory windows only (CUDA IPC over NVLink; also ranks
        sharing one GPU) -- the device-driven exchange, no NCCL.
    transport="nccl": NCCL communicator only (rank 0 creates the id).
    transport="auto": both; compares use the windows when max_report <=
        max_report_cap and fall back to NCCL otherwise (or if mapping fails).
    """
    import torch
    import torch.distributed as dist

    if transport not in ("peer", "nccl", "auto"):
        raise ValueError(f"unknown transport {transport!r}")
    rank, world = dist.get_rank(group), dist.get_world_size(group)
    uid = None
    if transport in ("nccl", "auto"):
        obj = [arc_verify_get_unique_id() if rank == 0 else None]
        dist.broadcast_object_list(obj, src=0, group=group)
        uid = obj[0]
    init(torch.cuda.current_device(), None, rank, world, uid)
    if transport == "nccl":
        return "nccl"
    h = arc_verify_peer_export(max_report_cap)
    handles = [None] * world
    dist.all_gather_object(handles, h, group=group)
    try:
        arc_verify_peer_open(handles)
        ok = 1
    except ArcVerifyError:
        if transport == "peer":
            raise
        ok = 0
    # every rank must take the same path: agree on the outcome
    flags = [None] * world
    dist.all_gather_object(flags, ok, group=group)
    if not all(flags):
        if transport == "peer":
            raise RuntimeError("peer windows could not be mapped on every rank")
        arc_verify_peer_export(0)  # drops the windows: the peer path stays off, NCCL is used
        return "nccl"
    return "peer"


def finalize() -> None:
    if _state["init"]:
        arc_verify_finalize()
        _state["init"] = False
        _state["nranks"] = 1


def _report_buffer(cap: int):
    arr = np.zeros(max(cap, 1), dtype=REPORT_DTYPE)
    return arr, arr.ctypes.data


_RES = arc_verify_result_t()  # reused: one context per process, calls are serialised
_compare_c = _lib.arc_verify_compare
_RES_REF = ctypes.byref(_RES)


def make_check(min_value: Optional[float] = None, bounds=None):
    """arc_verify_check_t for minValueToCheck and/or value bounds (lo, hi)."""
    if min_value is None and bounds is None:
        return None
    ck = arc_verify_check_t()
    if min_value is not None:
        ck.flags |= ARC_CHECK_MIN_VALUE
        ck.min_value = float(min_value)
    if bounds is not None:
        ck.flags |= ARC_CHECK_VALUE_BOUNDS
        ck.lo, ck.hi = float(bounds[0]), float(bounds[1])
    return ck


def compare(out, ref, abs_tol: float = 0.0, rel_tol: float = 0.0, max_report: int = 1 << 20,
            report=None, n: Optional[int] = None, min_value: Optional[float] = None, bounds=None) -> Result:
    """Verify ``out`` against ``ref`` (torch tensors, contiguous, same dtype).

    Tensors may live on the library's CUDA device or in (pinned) host memory.
    ``report``: optional preallocated buffer -- a numpy REPORT_DTYPE array (pinned
    if it comes from a pinned torch tensor) or a CUDA tensor of >= 24*cap bytes
    (then the report stays on the GPU).
    """
    if _TORCH_CODES is None:
        dtype_code(out)
    code = _TORCH_CODES.get(out.dtype)
    if code is None or out.dtype != ref.dtype:
        raise TypeError(f"unsupported or mismatched dtypes {out.dtype} / {ref.dtype}")
    if n is None:
        n = out.numel()
        if ref.numel() != n:
            raise ValueError("size mismatch")
    if n and not (out.is_contiguous() and ref.is_contiguous()):
        raise ValueError("tensors must be contiguous")
    if report is None:
        # sharded: the global report may exceed the local shard's length
        rep_arr, rep_ptr = _report_buffer(int(max_report) if _state["nranks"] > 1 else min(int(max_report), n))
    elif isinstance(report, np.ndarray):
        rep_arr, rep_ptr = report, report.ctypes.data
    else:
        rep_arr, rep_ptr = report, report.data_ptr()
    res = _RES
    res.report = rep_ptr if max_report > 0 else None
    ck = make_check(min_value, bounds)
    if ck is None:
        st = _compare_c(out.data_ptr() if n else None, ref.data_ptr() if n else None, n, code,
                        abs_tol, rel_tol, max_report, _RES_REF)
    else:
        st = _lib.arc_verify_compare_ex(out.data_ptr() if n else None, ref.data_ptr() if n else None, n, code,
                                        abs_tol, rel_tol, max_report, ctypes.byref(ck), _RES_REF)
    if st:
        raise ArcVerifyError(st, "arc_verify_compare")
    nr = res.n_reported
    rep = rep_arr[:nr] if isinstance(rep_arr, np.ndarray) else rep_arr
    return Result(res.n, res.n_mismatch, res.max_abs_err, res.max_rel_err, nr, rep)


class Prepared:
    """A comparison whose arguments are validated and marshalled once.

    ``p = prepare(out, ref, abs_tol, rel_tol, max_report, report=...)`` then each
    ``p()`` is one arc_verify_compare(_ex) call through pre-built ctypes
    arguments -- for callers that verify the same buffers repeatedly (an
    iterative solver checked every step; a benchmark loop).  The tensors and the
    report buffer must stay alive and in place.
    """

    __slots__ = ("_fn", "_args", "_res", "_rep", "_keep")

    def __init__(self, out, ref, abs_tol=0.0, rel_tol=0.0, max_report=1 << 20, report=None, n=None,
                 min_value=None, bounds=None):
        if _TORCH_CODES is None:
            dtype_code(out)
        code = _TORCH_CODES.get(out.dtype)
        if code is None or out.dtype != ref.dtype:
            raise TypeError(f"unsupported or mismatched dtypes {out.dtype} / {ref.dtype}")
        if n is None:
            n = out.numel()
            if ref.numel() != n:
                raise ValueError("size mismatch")
        if n and not (out.is_contiguous() and ref.is_contiguous()):
            raise ValueError("tensors must be contiguous")
        if report is None:
            report, ptr = _report_buffer(int(max_report) if _state["nranks"] > 1 else min(int(max_report), n))
        elif isinstance(report, np.ndarray):
            ptr = report.ctypes.data
        else:
            ptr = report.data_ptr()
        self._rep = report
        self._res = arc_verify_result_t()
        self._res.report = ptr if max_report > 0 else None
        ck = make_check(min_value, bounds)
        args = [ctypes.c_void_p(out.data_ptr() if n else None), ctypes.c_void_p(ref.data_ptr() if n else None),
                ctypes.c_uint64(n), ctypes.c_int(code), ctypes.c_double(abs_tol), ctypes.c_double(rel_tol),
                ctypes.c_uint64(max_report)]
        if ck is None:
            self._fn = _lib.arc_verify_compare
        else:
            self._fn = _lib.arc_verify_compare_ex
            args.append(ctypes.byref(ck))
        args.append(ctypes.byref(self._res))
        self._args = tuple(args)
        self._keep = (out, ref, ck)

    def __call__(self) -> Result:
        st = self._fn(*self._args)
        if st:
            raise ArcVerifyError(st, "arc_verify_compare")
        r = self._res
        nr = r.n_reported
        rep = self._rep[:nr] if isinstance(self._rep, np.ndarray) else self._rep
        return Result(r.n, r.n_mismatch, r.max_abs_err, r.max_rel_err, nr, rep)


def prepare(out, ref, abs_tol: float = 0.0, rel_tol: float = 0.0, max_report: int = 1 << 20, report=None,
            n: Optional[int] = None, min_value: Optional[float] = None, bounds=None) -> Prepared:
    """Validate and marshal a comparison once; call the result to run it (see Prepared)."""
    return Prepared(out, ref, abs_tol, rel_tol, max_report, report, n, min_value, bounds)


class PreparedBatch:
    """``pb = prepare_batch(regions)``: arc_verify_batch with the region table,
    result structs and report buffers built once; each ``pb()`` is one C call
    (one grid over every region).  Tensors must stay alive and in place."""

    __slots__ = ("_regs", "_res", "_reps", "_n", "_keep")

    def __init__(self, regions, report_buffers=None):
        regions = list(regions)
        R = len(regions)
        self._n = R
        self._regs = (arc_verify_region_t * R)()
        self._res = (arc_verify_result_t * R)()
        self._reps, keep = [], []
        for k, reg in enumerate(regions):
            out, ref, at, rt, mr = reg[:5]
            name = reg[5] if len(reg) > 5 else None
            n = out.numel()
            if ref.numel() != n or out.dtype != ref.dtype:
                raise ValueError(f"region {k}: size/dtype mismatch")
            if n and not (out.is_contiguous() and ref.is_contiguous()):
                raise ValueError(f"region {k}: tensors must be contiguous")
            if report_buffers is not None and report_buffers[k] is not None:
                arr = report_buffers[k]
                ptr = arr.ctypes.data if isinstance(arr, np.ndarray) else arr.data_ptr()
            else:
                arr, ptr = _report_buffer(min(int(mr), n))
            nm = name.encode() if name else None
            ck = reg[6] if len(reg) > 6 else None
            self._regs[k] = arc_verify_region_t(out.data_ptr() if n else None, ref.data_ptr() if n else None, n,
                                                dtype_code(out), float(at), float(rt), int(mr), nm,
                                                ctypes.pointer(ck) if ck is not None else None)
            self._res[k].report = ptr if mr > 0 else None
            self._reps.append(arr)
            keep.append((out, ref, nm, ck))
        self._keep = keep

    def __call__(self) -> list[Result]:
        _check(_lib.arc_verify_batch(self._regs, self._n, self._res), "arc_verify_batch")
        outs = []
        for k in range(self._n):
            r = self._res[k]
            nr = int(r.n_reported)
            rep = self._reps[k][:nr] if isinstance(self._reps[k], np.ndarray) else self._reps[k]
            outs.append(Result(int(r.n), int(r.n_mismatch), float(r.max_abs_err), float(r.max_rel_err), nr, rep))
        return outs


def prepare_batch(regions, report_buffers=None) -> PreparedBatch:
    """Validate and marshal a batch once (see PreparedBatch)."""
    return PreparedBatch(regions, report_buffers)


def batch(regions, options: Optional[str] = None, select: bool = False) -> list[Result]:
    """regions: iterable of (out, ref, abs_tol, rel_tol, max_report[, name[, check]]) with torch
    tensors; ``check`` is an arc_verify_check_t (see make_check) or None."""
    regions = list(regions)
    R = len(regions)
    regs = (arc_verify_region_t * R)()
    results = (arc_verify_result_t * R)()
    keep, keep_ck = [], []
    for k, reg in enumerate(regions):
        out, ref, at, rt, mr = reg[:5]
        name = reg[5] if len(reg) > 5 else None
        n = out.numel()
        if ref.numel() != n or out.dtype != ref.dtype:
            raise ValueError(f"region {k}: size/dtype mismatch")
        arr, ptr = _report_buffer(min(int(mr), n))
        keep.append(arr)
        nm = name.encode() if name else None
        keep.append(nm)
        ck = reg[6] if len(reg) > 6 else None
        regs[k] = arc_verify_region_t(out.data_ptr() if n else None, ref.data_ptr() if n else None, n,
                                      dtype_code(out), float(at), float(rt), int(mr), nm,
                                      ctypes.pointer(ck) if ck is not None else None)
        if ck is not None:
            keep_ck.append(ck)
        results[k].report = ptr if mr > 0 else None
    if select or options is not None:
        sel = (ctypes.c_uint8 * R)()
        st = _lib.arc_verify_batch_selected(regs, R, options.encode() if options is not None else None, results,
                                            ctypes.cast(sel, ctypes.c_void_p))
        _check(st, "arc_verify_batch_selected")
    else:
        arc_verify_batch(regs, results)
    outs = []
    for k in range(R):
        r = results[k]
        outs.append(Result(int(r.n), int(r.n_mismatch), float(r.max_abs_err), float(r.max_rel_err),
                           int(r.n_reported), keep[2 * k][: r.n_reported]))
    return outs
