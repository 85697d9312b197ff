"""CPU oracle for the kernel-verification result comparison -- TEST INFRASTRUCTURE.

Only ``tests/``, ``__graft_entry__.smoke()`` and the ``cpu_baseline`` /
``--impl reference`` legs of ``bench.py`` may import this package.  The product
package ``paper_conf_ipps_leelv14_b200`` never imports it and shares no code
with it.

``compare`` wraps ``arc_oracle.c`` (the plain, sequential per-element
definition; see the header of that file for the PAPER.md passages it follows:
P:159, sec. III-A).  ``merge_shards`` is the plain
definition of the cross-GPU merge (SURVEY.md sec. 8(a) a8 / DESIGN.md sec. 3,
reading R-shard): the global result of p contiguous shards is the sum of the
counts, the max of the maxima, and the concatenation of the per-shard reports
in rank order with global indices, truncated to ``max_report``.  The paper
itself is single-GPU; the merge is a reading, pinned in tests by
checking it against the unsharded oracle.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from dataclasses import dataclass, field

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "arc_oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")

DTYPES = {"f32": 0, "f64": 1, "i32": 2, "i64": 3, "u8": 4}
NP_DTYPES = {"f32": np.float32, "f64": np.float64, "i32": np.int32, "i64": np.int64, "u8": np.uint8}

CFLAGS = ["-O2", "-std=c99", "-ffp-contract=off", "-fno-fast-math", "-fPIC", "-shared"]


def build(force: bool = False) -> str:
    """Compile arc_oracle.c with gcc (no FMA contraction, no fast-math)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", *CFLAGS, "-o", tmp, _SRC, "-lm"])
        os.replace(tmp, _LIB)
    return _LIB


class _Mismatch(ctypes.Structure):
    _fields_ = [("index", ctypes.c_uint64), ("out_bits", ctypes.c_uint64), ("ref_bits", ctypes.c_uint64)]


class _Result(ctypes.Structure):
    _fields_ = [
        ("n", ctypes.c_uint64),
        ("n_mismatch", ctypes.c_uint64),
        ("max_abs_err", ctypes.c_double),
        ("max_rel_err", ctypes.c_double),
        ("n_reported", ctypes.c_uint64),
    ]


_lib = None


def _load():
    global _lib
    if _lib is None:
        lib = ctypes.CDLL(build())
        lib.oracle_compare.restype = ctypes.c_int
        lib.oracle_compare.argtypes = [
            ctypes.c_void_p, ctypes.c_void_p, ctypes.c_uint64, ctypes.c_int,
            ctypes.c_double, ctypes.c_double, ctypes.c_uint64,
            ctypes.c_void_p, ctypes.POINTER(_Result),
        ]
        lib.oracle_compare_ex.restype = ctypes.c_int
        lib.oracle_compare_ex.argtypes = [
            ctypes.c_void_p, ctypes.c_void_p, ctypes.c_uint64, ctypes.c_int,
            ctypes.c_double, ctypes.c_double, ctypes.c_uint64,
            ctypes.c_int, ctypes.c_double, ctypes.c_double, ctypes.c_double,
            ctypes.c_void_p, ctypes.POINTER(_Result),
        ]
        lib.oracle_checksum.restype = ctypes.c_int
        lib.oracle_checksum.argtypes = [ctypes.c_void_p, ctypes.c_uint64, ctypes.POINTER(ctypes.c_uint64)]
        lib.oracle_sizeof_result.restype = ctypes.c_size_t
        lib.oracle_sizeof_mismatch.restype = ctypes.c_size_t
        assert lib.oracle_sizeof_result() == ctypes.sizeof(_Result)
        assert lib.oracle_sizeof_mismatch() == 24
        _lib = lib
    return _lib


REPORT_DTYPE = np.dtype([("index", "<u8"), ("out_bits", "<u8"), ("ref_bits", "<u8")])


@dataclass
class OracleResult:
    n: int
    n_mismatch: int
    max_abs_err: float
    max_rel_err: float
    n_reported: int
    report: np.ndarray = field(repr=False)  # structured REPORT_DTYPE, length n_reported


class OracleError(ValueError):
    pass


def compare(out, ref, dtype: str, abs_tol: float, rel_tol: float, max_report: int,
            min_value=None, bounds=None) -> OracleResult:
    """Run the sequential oracle on two host arrays (numpy, contiguous).

    ``min_value`` (minValueToCheck) and ``bounds`` = (lo, hi) (value-bound
    directives) select oracle_compare_ex (NEXT row N2).
    """
    lib = _load()
    npdt = NP_DTYPES[dtype]
    out = np.ascontiguousarray(out, dtype=npdt).reshape(-1)
    ref = np.ascontiguousarray(ref, dtype=npdt).reshape(-1)
    if out.shape != ref.shape:
        raise OracleError("shape mismatch")
    n = out.size
    cap = min(int(max_report), n)
    report = np.zeros(max(cap, 1), dtype=REPORT_DTYPE)
    res = _Result()
    if min_value is None and bounds is None:
        st = lib.oracle_compare(
            out.ctypes.data if n else None, ref.ctypes.data if n else None, n, DTYPES[dtype],
            float(abs_tol), float(rel_tol), int(max_report),
            report.ctypes.data if max_report > 0 else None, ctypes.byref(res),
        )
    else:
        flags = (1 if min_value is not None else 0) | (2 if bounds is not None else 0)
        lo, hi = bounds if bounds is not None else (0.0, 0.0)
        st = lib.oracle_compare_ex(
            out.ctypes.data if n else None, ref.ctypes.data if n else None, n, DTYPES[dtype],
            float(abs_tol), float(rel_tol), int(max_report),
            flags, float(min_value if min_value is not None else 0.0), float(lo), float(hi),
            report.ctypes.data if max_report > 0 else None, ctypes.byref(res),
        )
    if st != 0:
        raise OracleError("oracle_compare rejected its arguments")
    return OracleResult(int(res.n), int(res.n_mismatch), float(res.max_abs_err),
                        float(res.max_rel_err), int(res.n_reported), report[: res.n_reported].copy())


def merge_shards(parts, max_report: int) -> OracleResult:
    """Plain definition of the cross-shard merge (reading R-shard).

    ``parts`` is a list, in rank order, of OracleResult computed on contiguous
    shards [off_r, off_r + n_r).  Global index = local index + sum of n over
    lower ranks.
    """
    n = sum(p.n for p in parts)
    count = sum(p.n_mismatch for p in parts)
    max_abs = max([p.max_abs_err for p in parts] + [0.0])
    max_rel = max([p.max_rel_err for p in parts] + [0.0])
    entries = []
    off = 0
    for p in parts:
        rep = p.report.copy()
        rep["index"] += np.uint64(off)
        entries.append(rep)
        off += p.n
    report = np.concatenate(entries) if entries else np.zeros(0, dtype=REPORT_DTYPE)
    n_rep = min(count, int(max_report))
    return OracleResult(n, count, max_abs, max_rel, n_rep, report[:n_rep].copy())


def compare_threads(out, ref, dtype: str, abs_tol: float, rel_tol: float, max_report: int,
                    threads: int | None = None, pool=None) -> OracleResult:
    """The sequential oracle, unchanged, on ``threads`` contiguous chunks at once
    (host threads: ctypes releases the GIL during each call), merged by
    ``merge_shards`` -- the same definition as the cross-GPU merge.  Equal to
    ``compare`` on the whole arrays (pinned in tests/test_oracle.py).  Used only
    to time the oracle on all host cores (bench.py cpu_baseline / --impl
    reference)."""
    from concurrent.futures import ThreadPoolExecutor

    out = np.ascontiguousarray(out).reshape(-1)
    ref = np.ascontiguousarray(ref).reshape(-1)
    threads = max(1, int(threads or len(os.sched_getaffinity(0))))
    n = out.size
    cuts = [k * n // threads for k in range(threads + 1)]

    def part(k):
        return compare(out[cuts[k]:cuts[k + 1]], ref[cuts[k]:cuts[k + 1]], dtype, abs_tol, rel_tol, max_report)

    if pool is not None:
        parts = list(pool.map(part, range(threads)))
    else:
        with ThreadPoolExecutor(threads) as ex:
            parts = list(ex.map(part, range(threads)))
    return merge_shards(parts, max_report)


def checksum(data) -> tuple[int, int]:
    """The N4 debug-assertion checksum (sum, xor) of a host array's bytes."""
    lib = _load()
    b = np.ascontiguousarray(data).reshape(-1).view(np.uint8)
    out = (ctypes.c_uint64 * 2)()
    if lib.oracle_checksum(b.ctypes.data if b.size else None, b.size, out) != 0:
        raise OracleError("oracle_checksum rejected its arguments")
    return int(out[0]), int(out[1])
