"""The five BASELINE.json configurations as seeded synthetic workloads.

Shapes and value distributions follow SURVEY.md sec. 8(d) / DESIGN.md sec. 4.
Each workload yields (out, ref) for any element range, so shards and chunks
are generated independently and bit-identically on CPU or CUDA.  ``planted``
lists the indices where the generator put a mismatch by construction (the
closed-form pin for the oracle's count and report).
"""
from __future__ import annotations

from dataclasses import dataclass, field

import torch

from . import (S_INJECT, add_ulp_noise, distinct_indices, f32_field, f32_uniform,
               f64_values, hash64_py, i32_values, substream)

__all__ = ["Region", "C1", "C2", "C3_REGIONS", "C4", "C5", "c3_regions", "CONFIGS",
           "C1_SPECIALS", "TORCH_DTYPES"]

TORCH_DTYPES = {"f32": torch.float32, "f64": torch.float64, "i32": torch.int32,
                "i64": torch.int64, "u8": torch.uint8}

_NAN = float("nan")
_INF = float("inf")

# (index, out, ref, is_mismatch) -- SURVEY.md sec. 8(d) row C1; the match column
# is the hand-worked reading of rules 1-5.
C1_SPECIALS = [
    (0, _NAN, _NAN, False),
    (1, _NAN, 1.0, True),
    (2, 1.0, _NAN, True),
    (3, 0.0, -0.0, False),
    (4, -0.0, 0.0, False),
    (5, _INF, _INF, False),
    (6, -_INF, _INF, True),
    (7, 1e30, _INF, True),
    (8, _INF, 3e38, True),
    (9, 1.401298464324817e-45, 0.0, False),
    (10, 2e-6, 0.0, True),
    (11, 0.1384209543466568, 0.13841857016086578, True),
    (12, 1.00001, 1.0, False),
    (13, 1.0000115, 1.0, True),
]


@dataclass
class Region:
    """One verification region: a named (out, ref) pair and its tolerances."""

    name: str
    dtype: str
    n: int
    seed: int
    abs_tol: float
    rel_tol: float
    max_report: int
    kind: str  # value recipe
    n_inject: int = 0
    n_nan: int = 0
    extra: dict = field(default_factory=dict)

    # ------------------------------------------------------------ construction
    def _inject_idx(self) -> list[int]:
        lo = 16 if self.kind == "c1" else 0
        k = self.n_inject + self.n_nan
        return distinct_indices(substream(self.seed, S_INJECT), k, lo, self.n) if k else []

    def injected(self) -> list[int]:
        return self._inject_idx()[: self.n_inject]

    def nan_pairs(self) -> list[int]:
        return self._inject_idx()[self.n_inject:]

    def planted(self) -> list[int]:
        """Sorted indices that mismatch by construction."""
        s = set(self._inject_idx())
        if self.kind == "c1":
            s |= {i for (i, _o, _r, mis) in C1_SPECIALS if mis}
        if self.kind == "c2" and self.extra.get("variant") == "B":
            row = 8190
            s |= {row * 8192 + j for j in range(1, 8191)}
        return sorted(s)

    def slice(self, start: int = 0, count: int | None = None, device="cpu"):
        """(out, ref) for elements [start, start+count)."""
        if count is None:
            count = self.n - start
        assert 0 <= start and start + count <= self.n
        dev = torch.device(device)
        if self.kind in ("c1", "f32"):
            ref = f32_uniform(self.seed, start, count, dev)
            out = add_ulp_noise(ref, self.seed, start)
        elif self.kind == "c2":
            ref = f32_field(self.seed, start, count, dev)
            out = add_ulp_noise(ref, self.seed, start)
        elif self.kind == "f64":
            ref = f64_values(self.seed, start, count, dev)
            out = add_ulp_noise(ref, self.seed, start)
        elif self.kind == "i32":
            ref = i32_values(self.seed, start, count, dev)
            out = ref.clone()
        elif self.kind == "c5":
            ref = i32_values(self.seed, start, count, dev)
            par = (torch.arange(start, start + count, dtype=torch.int64, device=dev) & 1).to(torch.int32)
            out = ref ^ par
        else:
            raise ValueError(self.kind)
        self._apply_planted(out, ref, start, count)
        return out, ref

    def _apply_planted(self, out, ref, start, count):
        end = start + count
        for i in self.injected():
            if start <= i < end:
                j = i - start
                if self.dtype == "f32":
                    if self.kind == "c2":
                        out[j] = (ref[j:j + 1].view(torch.int32) ^ (1 << 22)).view(torch.float32)[0]
                    else:
                        r = ref[j]
                        out[j] = r - 0.5 if r >= 0 else r + 0.5
                elif self.dtype == "f64":
                    out[j] = (ref[j:j + 1].view(torch.int64) ^ (1 << 50)).view(torch.float64)[0]
                elif self.dtype == "i32":
                    out[j] = ref[j] ^ 1
        for i in self.nan_pairs():
            if start <= i < end:
                out[i - start] = _NAN
        if self.kind == "c1":
            for (i, o, r, _mis) in C1_SPECIALS:
                if start <= i < end:
                    out[i - start] = o
                    ref[i - start] = r
        if self.kind == "c2" and self.extra.get("variant") == "B":
            row0 = 8190 * 8192
            lo, hi = max(start, row0 + 1), min(end, row0 + 8191)
            if lo < hi:
                seg = ref[lo - start:hi - start]
                out[lo - start:hi - start] = (seg.view(torch.int32) ^ (1 << 22)).view(torch.float32)


# ------------------------------------------------------------------- configs
def C1() -> Region:
    """fp32, 2^20 elements, 37 injected + NaN/+-0/Inf specials (BASELINE configs[0])."""
    return Region("C1", "f32", 1 << 20, 2015, 1e-6, 1e-5, 1 << 20, "c1", n_inject=37)


def C2(variant: str = "A") -> Region:
    """Jacobi-2D 8192x8192 fp32 output vs reference, rel 1e-5, abs 0 (configs[1])."""
    return Region(f"C2{variant}", "f32", 8192 * 8192, 2016, 0.0, 1e-5, 1 << 20, "c2",
                  extra={"variant": variant})


# (name, dtype, shape) -- the twelve apps of P:299-303; shapes are the public
# suites' largest standard inputs (a proposal; the paper states none).
C3_REGIONS = [
    ("BACKPROP", "f32", (65537, 17)),
    ("BFS", "i32", (1000000,)),
    ("CFD", "f32", (232536, 5)),
    ("CG", "f64", (150002,)),
    ("EP", "f64", (12,)),
    ("HOTSPOT", "f32", (1024, 1024)),
    ("JACOBI", "f32", (8192, 8192)),
    ("KMEANS", "i32", (494020,)),
    ("LUD", "f32", (2048, 2048)),
    ("NW", "i32", (2049, 2049)),
    ("SPMUL", "f32", (2000003,)),
    ("SRAD", "f32", (2048, 2048)),
]


def c3_regions() -> list[Region]:
    """Twelve benchmark-shaped region outputs, mixed f32/f64/i32 (configs[2])."""
    regs = []
    for k, (name, dt, shape) in enumerate(C3_REGIONS):
        n = 1
        for s in shape:
            n *= s
        seed = substream(2017, 100 + k)
        n_inj = hash64_py(seed, 77) % 6
        tol = (0.0, 0.0) if dt == "i32" else (1e-6, 1e-5)
        regs.append(Region(name, dt, n, seed, tol[0], tol[1], 1024, dt, n_inject=n_inj,
                           extra={"shape": shape}))
    return regs


def C4(n: int = 1 << 29) -> Region:
    """fp64 2^29 elements (4 GiB per array), 512 injected + 4 NaN pairs (configs[3])."""
    return Region("C4", "f64", n, 2018, 1e-6, 1e-5, 1 << 20, "f64", n_inject=512, n_nan=4)


def C5(n: int = 1 << 30) -> Region:
    """int32 2^30 elements, out = ref ^ (i & 1): 50% mismatches, max_report 2^20 (configs[4])."""
    return Region("C5", "i32", n, 2019, 0.0, 0.0, 1 << 20, "c5")


CONFIGS = {"C1": C1, "C2": C2, "C4": C4, "C5": C5}
