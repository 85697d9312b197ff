"""Pins for the CPU oracle (runs without a GPU).

Every pin comes from something other than the oracle itself: hand-worked values
(tests/golden/hand_table.txt), numpy's isclose / nanmax as the textbook
routine, exact rational arithmetic, closed forms of the generator's planted
mismatches, brute force over special values, and invariants.
"""
import math
import os
from fractions import Fraction

import numpy as np
import pytest
import torch

import synth

GOLDEN = os.path.join(os.path.dirname(__file__), "golden", "hand_table.txt")


def f32(bits):
    return np.array(bits, dtype=np.uint32).view(np.float32)


def rn_div(d: float, y: float) -> float:
    """Correctly rounded d/|y| via exact rationals (independent of C division)."""
    q = Fraction(d) / abs(Fraction(y))
    return float(q)  # Fraction -> float rounds to nearest-even


# ------------------------------------------------------------------ golden table
def _golden_rows():
    rows = []
    for line in open(GOLDEN):
        line = line.split("#", 1)[0].strip()
        if not line:
            continue
        ob, rb, at, rt, mis, d, r = line.split()
        rows.append((int(ob, 16), int(rb, 16), float(at), float(rt), int(mis), d, r))
    return rows


@pytest.mark.parametrize("row", _golden_rows())
def test_golden_hand_table(oracle_mod, row):
    ob, rb, at, rt, mis, d, r = row
    out, ref = f32([ob]), f32([rb])
    res = oracle_mod.compare(out, ref, "f32", at, rt, 4)
    assert res.n_mismatch == mis
    assert res.n_reported == mis
    if mis:
        e = res.report[0]
        assert (int(e["index"]), int(e["out_bits"]), int(e["ref_bits"])) == (0, ob, rb)
    if d == "undef":
        assert res.max_abs_err == 0.0 and res.max_rel_err == 0.0
        return
    dv = float(d)
    assert res.max_abs_err == dv
    if r == "frac":
        rv = rn_div(dv, float(ref[0]))
    else:
        rv = float(r)
    assert res.max_rel_err == rv


def test_sentinel_needs_fp64():
    """The sentinel pair decides differently in fp32 and fp64 (reading R3)."""
    x, y = np.float32(0.1384209543466568), np.float32(0.13841857016086578)
    d32 = abs(x - y)
    t32 = np.float32(1e-6) + np.float32(1e-5) * abs(y)
    assert d32 <= t32  # fp32 evaluation would call it a match
    d64 = abs(float(x) - float(y))
    t64 = 1e-6 + 1e-5 * abs(float(y))
    assert d64 > t64  # fp64 evaluation (the reading) calls it a mismatch


# ------------------------------------------------------- brute force vs numpy
def _numpy_expect(out, ref, at, rt):
    x = out.astype(np.float64)
    y = ref.astype(np.float64)
    with np.errstate(all="ignore"):
        match = np.isclose(x, y, rtol=rt, atol=at, equal_nan=True)
        d = np.where(x == y, 0.0, np.abs(x - y))
        r = np.where(x == y, 0.0, np.where(np.isinf(y), np.inf, d / np.abs(y)))
    valid = ~(np.isnan(x) | np.isnan(y))
    dmax = float(np.max(d[valid])) if valid.any() else 0.0
    rmax = float(np.max(r[valid])) if valid.any() else 0.0
    return match, max(dmax, 0.0), max(rmax, 0.0)


@pytest.mark.parametrize("tol", synth.TOL_PAIRS)
def test_bruteforce_special_pairs(oracle_mod, tol):
    at, rt = tol
    sp = f32(synth.F32_SPECIAL_BITS)
    out = np.repeat(sp, sp.size)
    ref = np.tile(sp, sp.size)
    match, dmax, rmax = _numpy_expect(out, ref, at, rt)
    res = oracle_mod.compare(out, ref, "f32", at, rt, out.size)
    exp_idx = np.flatnonzero(~match)
    assert res.n_mismatch == exp_idx.size
    assert np.array_equal(res.report["index"], exp_idx.astype(np.uint64))
    assert np.array_equal(res.report["out_bits"], out.view(np.uint32)[exp_idx].astype(np.uint64))
    assert np.array_equal(res.report["ref_bits"], ref.view(np.uint32)[exp_idx].astype(np.uint64))
    assert res.max_abs_err == dmax
    assert res.max_rel_err == rmax


def _boundary_pairs(rng, n, dtype):
    if dtype == "f32":
        ref = rng.uniform(-4, 4, n).astype(np.float32)
        ref[::17] = 0
        k = rng.integers(-140, 140, n).astype(np.int64)
        bits = ref.view(np.int32).astype(np.int64) + np.where(ref == 0, 0, k)
        out = bits.astype(np.int32).view(np.float32).copy()
        out[::23] = rng.uniform(-2e-6, 2e-6, out[::23].size).astype(np.float32)
    else:
        ref = rng.uniform(-4, 4, n)
        ref[::17] = 0
        k = rng.integers(-1 << 34, 1 << 34, n)
        out = (ref.view(np.int64) + np.where(ref == 0, 0, k)).view(np.float64).copy()
        out[::23] = rng.uniform(-2e-6, 2e-6, out[::23].size)
    return out, ref


@pytest.mark.parametrize("dtype", ["f32", "f64"])
@pytest.mark.parametrize("tol", [(1e-6, 1e-5), (0.0, 1e-5), (1e-6, 0.0)])
def test_boundary_random_vs_numpy(oracle_mod, dtype, tol):
    rng = np.random.default_rng(7)
    out, ref = _boundary_pairs(rng, 200_003, dtype)
    at, rt = tol
    match, dmax, rmax = _numpy_expect(out, ref, at, rt)
    exp_idx = np.flatnonzero(~match)
    assert 0 < exp_idx.size < out.size  # the set straddles the boundary
    for max_report in (0, 1, 100, exp_idx.size, 10 ** 9):
        res = oracle_mod.compare(out, ref, dtype, at, rt, max_report)
        assert res.n_mismatch == exp_idx.size
        assert res.n_reported == min(exp_idx.size, max_report)
        assert np.array_equal(res.report["index"], exp_idx[: res.n_reported].astype(np.uint64))
        assert res.max_abs_err == dmax
        assert res.max_rel_err == rmax


def test_ulp_window_boundary(oracle_mod):
    """Every fp32 out within +-128 ulps of fixed refs: the first mismatch ulp is the closed form."""
    refs = np.array([1.0, 0.75, -3.0, 1e-3, 12345.0], dtype=np.float32)
    for y in refs:
        k = np.arange(-128, 129)
        out = (np.int64(np.float32(y).view(np.int32)) + k).astype(np.int32).view(np.float32)
        ref = np.full(out.size, y, dtype=np.float32)
        res = oracle_mod.compare(out, ref, "f32", 1e-6, 1e-5, 1000)
        t = Fraction(1e-6) + Fraction(1e-5) * abs(Fraction(float(y)))  # exact margin
        # the fp64 margin is t rounded twice; away from rounding ties the decision equals
        # the exact comparison |x - y| <= t, which these refs never hit.
        exp = [i for i, x in enumerate(out) if abs(Fraction(float(x)) - Fraction(float(y))) > t]
        assert list(res.report["index"]) == exp


# --------------------------------------------------------------- integer forms
def test_integer_closed_forms(oracle_mod):
    n = 1 << 16
    c5 = synth.C5(n)
    out, ref = c5.slice(0, n)
    res = oracle_mod.compare(out.numpy(), ref.numpy(), "i32", 0, 0, 1 << 12)
    assert res.n_mismatch == n // 2
    assert np.array_equal(res.report["index"], np.arange(1, 2 * (1 << 12), 2, dtype=np.uint64))
    assert res.max_abs_err == 1.0 and res.max_rel_err == 0.0
    # extremes: |INT_MIN - INT_MAX| exactly, then RN to double
    a = np.array([np.iinfo(np.int32).min, 5, 7], dtype=np.int32)
    b = np.array([np.iinfo(np.int32).max, 5, -7], dtype=np.int32)
    res = oracle_mod.compare(a, b, "i32", 0.5, 0.5, 8)  # tolerances ignored for ints
    assert res.n_mismatch == 2 and res.max_abs_err == float(2 ** 32 - 1)
    assert list(res.report["out_bits"]) == [0x80000000, 7]  # zero-extended raw bits
    assert list(res.report["ref_bits"]) == [0x7FFFFFFF, 0xFFFFFFF9]
    a = np.array([np.iinfo(np.int64).min, 1], dtype=np.int64)
    b = np.array([np.iinfo(np.int64).max, 1], dtype=np.int64)
    res = oracle_mod.compare(a, b, "i64", 0, 0, 8)
    assert res.n_mismatch == 1 and res.max_abs_err == float(2 ** 64)  # 2^64-1 rounds to 2^64
    a = np.array([0, 255, 3], dtype=np.uint8)
    b = np.array([255, 0, 3], dtype=np.uint8)
    res = oracle_mod.compare(a, b, "u8", 0, 0, 8)
    assert res.n_mismatch == 2 and res.max_abs_err == 255.0
    assert list(res.report["index"]) == [0, 1]


# ------------------------------------------------------- planted closed forms
def test_c1_planted(oracle_mod):
    c1 = synth.C1()
    out, ref = c1.slice()
    res = oracle_mod.compare(out.numpy(), ref.numpy(), "f32", c1.abs_tol, c1.rel_tol, c1.max_report)
    planted = c1.planted()
    assert len(planted) == 45
    assert res.n_mismatch == 45
    assert list(res.report["index"]) == planted
    assert math.isinf(res.max_abs_err) and math.isinf(res.max_rel_err)


@pytest.mark.slow
def test_c2_variants_planted(oracle_mod):
    for v in ("A", "B"):
        c2 = synth.C2(v)
        out, ref = c2.slice()
        res = oracle_mod.compare(out.numpy(), ref.numpy(), "f32", c2.abs_tol, c2.rel_tol, c2.max_report)
        assert list(res.report["index"]) == c2.planted()
        if v == "A":
            assert res.n_mismatch == 0
            assert 0 < res.max_abs_err <= 4 * 2.0 ** -23  # <= 4 ulps of [1, 1.5)
        else:
            assert res.n_mismatch == 8190
            assert res.max_abs_err == 0.5


def test_c3_planted(oracle_mod):
    for reg in synth.c3_regions():
        if reg.n > 5_000_000:
            continue  # JACOBI is C2-sized; covered by the slow test above
        out, ref = reg.slice()
        res = oracle_mod.compare(out.numpy(), ref.numpy(), reg.dtype, reg.abs_tol, reg.rel_tol, reg.max_report)
        assert list(res.report["index"]) == reg.planted(), reg.name
        assert res.n_mismatch == reg.n_inject


def test_c4_chunk_planted(oracle_mod):
    c4 = synth.C4()
    lo, cnt = 0, 1 << 22
    out, ref = c4.slice(lo, cnt)
    res = oracle_mod.compare(out.numpy(), ref.numpy(), "f64", c4.abs_tol, c4.rel_tol, c4.max_report)
    exp = [i for i in c4.planted() if lo <= i < lo + cnt]
    assert list(res.report["index"]) == exp


# ------------------------------------------------------------ invariants/edges
def test_edges(oracle_mod):
    e = np.zeros(0, dtype=np.float32)
    res = oracle_mod.compare(e, e, "f32", 1e-6, 1e-5, 10)
    assert (res.n, res.n_mismatch, res.max_abs_err, res.max_rel_err, res.n_reported) == (0, 0, 0.0, 0.0, 0)
    a = f32(synth.F32_SPECIAL_BITS)
    res = oracle_mod.compare(a, a, "f32", 0, 0, 10)  # aliasing: everything matches itself
    assert res.n_mismatch == 0 and res.max_abs_err == 0.0
    b = a.copy()
    b[3] = 5.0
    res = oracle_mod.compare(a, b, "f32", 0, 0, 0)  # count only
    assert res.n_mismatch == 1 and res.n_reported == 0
    for bad in [(-1.0, 0.0), (0.0, float("nan")), (float("inf"), 0.0)]:
        with pytest.raises(oracle_mod.OracleError):
            oracle_mod.compare(a, b, "f32", bad[0], bad[1], 1)


# --------------------------------------------------------------- shard merge
@pytest.mark.parametrize("p", [2, 3, 4, 8])
@pytest.mark.parametrize("max_report", [0, 5, 20, 45, 1000])
def test_shard_merge_equals_unsharded(oracle_mod, p, max_report):
    c1 = synth.C1()
    out, ref = c1.slice()
    out, ref = out.numpy(), ref.numpy()
    full = oracle_mod.compare(out, ref, "f32", 1e-6, 1e-5, max_report)
    n = out.size
    cuts = [0] + sorted(synth.distinct_indices(99 + p, p - 1, 1, n)) + [n]
    parts = [oracle_mod.compare(out[a:b], ref[a:b], "f32", 1e-6, 1e-5, max_report)
             for a, b in zip(cuts[:-1], cuts[1:])]
    m = oracle_mod.merge_shards(parts, max_report)
    assert (m.n, m.n_mismatch, m.n_reported) == (full.n, full.n_mismatch, full.n_reported)
    assert m.max_abs_err == full.max_abs_err and m.max_rel_err == full.max_rel_err
    assert np.array_equal(m.report, full.report)


@pytest.mark.parametrize("threads", [1, 3, 8])
@pytest.mark.parametrize("max_report", [0, 7, 45, 1 << 20])
def test_threaded_oracle_equals_sequential(oracle_mod, threads, max_report):
    """compare_threads (the oracle on contiguous chunks in host threads + merge_shards, used
    only to time the oracle on all cores) returns exactly the sequential oracle's result."""
    for c, dt in ((synth.C1(), "f32"), (synth.C4(1 << 18), "f64"), (synth.C5(1 << 16), "i32")):
        out, ref = c.slice()
        out, ref = out.numpy(), ref.numpy()
        full = oracle_mod.compare(out, ref, dt, c.abs_tol, c.rel_tol, max_report)
        m = oracle_mod.compare_threads(out, ref, dt, c.abs_tol, c.rel_tol, max_report, threads=threads)
        assert (m.n, m.n_mismatch, m.n_reported) == (full.n, full.n_mismatch, full.n_reported)
        assert m.max_abs_err == full.max_abs_err and m.max_rel_err == full.max_rel_err
        assert np.array_equal(m.report, full.report)


# ---------------------------------------------------------------- generator
def test_generator_pinned_to_python():
    idx = torch.tensor([0, 1, 2, 3, 99991, (1 << 33) + 5], dtype=torch.int64)
    for seed in (2014, 2018, synth.substream(2015, 1)):
        h = synth.hash64(seed, idx).tolist()
        for i, v in zip(idx.tolist(), h):
            assert (v & synth.MASK64) == synth.hash64_py(seed, i)
    v = synth.f32_uniform(5, 0, 1 << 16)
    assert v.min() >= -1 and v.max() < 1
    assert torch.equal(v * 2 ** 23, torch.round(v * 2 ** 23))
    k = synth.noise_k(5, 0, 1 << 16)
    assert int(k.min()) == -4 and int(k.max()) == 4
    d = synth.f64_values(5, 0, 1 << 16).abs()
    assert float(d.min()) >= 2.0 ** -16 and float(d.max()) < 2.0 ** 16
    # shards regenerate bit-identically
    a = synth.C4().slice(1000, 5000)[0]
    b = synth.C4().slice(3000, 1000)[0]
    assert torch.equal(a[2000:3000].view(torch.int64), b.view(torch.int64))


# ------------------------------------------------- N2: minValueToCheck / bounds
def _numpy_expect_checks(out, ref, at, rt, min_value, bounds):
    """Library-routine pin for the optional checks (readings R10, R11)."""
    x = out.astype(np.float64)
    y = ref.astype(np.float64)
    with np.errstate(all="ignore"):
        match = np.isclose(x, y, rtol=rt, atol=at, equal_nan=True)
        d = np.where(x == y, 0.0, np.abs(x - y))
        r = np.where(x == y, 0.0, np.where(np.isinf(y), np.inf, d / np.abs(y)))
    keep = np.ones(x.size, dtype=bool)
    if min_value is not None:
        keep &= ~(np.abs(y) <= min_value)
    if bounds is not None:
        keep &= ~((~match) & (bounds[0] <= x) & (x <= bounds[1]))
    mis = (~match) & keep
    valid = keep & ~(np.isnan(x) | np.isnan(y))
    dmax = float(np.max(d[valid])) if valid.any() else 0.0
    rmax = float(np.max(r[valid])) if valid.any() else 0.0
    return np.flatnonzero(mis), dmax, rmax


@pytest.mark.parametrize("min_value,bounds", [(1e-32, None), (0.5, None), (None, (-0.25, 0.25)),
                                              (1e-3, (0.0, 1.0)), (0.0, (-np.inf, np.inf))])
def test_checks_vs_numpy(oracle_mod, min_value, bounds):
    rng = np.random.default_rng(3)
    out, ref = _boundary_pairs(rng, 100_003, "f32")
    sp = np.array(synth.F32_SPECIAL_BITS, dtype=np.uint32).view(np.float32)
    out = np.concatenate([out, np.repeat(sp, sp.size)])
    ref = np.concatenate([ref, np.tile(sp, sp.size)])
    idx, dmax, rmax = _numpy_expect_checks(out, ref, 1e-6, 1e-5, min_value, bounds)
    res = oracle_mod.compare(out, ref, "f32", 1e-6, 1e-5, 10 ** 6, min_value=min_value, bounds=bounds)
    assert res.n_mismatch == idx.size
    assert np.array_equal(res.report["index"], idx.astype(np.uint64))
    assert res.max_abs_err == dmax and res.max_rel_err == rmax


def test_checks_hand_cases(oracle_mod):
    """The paper's example minValueToCheck=1e-32 and a value bound."""
    out = np.array([1e-40, 5e-33, 3.0, 0.6, np.nan], dtype=np.float64)
    ref = np.array([0.0, 1e-33, 2.0, 0.5, 1.0], dtype=np.float64)
    # without checks: 1e-40 vs 0 matches (abs 1e-6); 5e-33 vs 1e-33 matches; 3 vs 2, 0.6 vs 0.5, NaN vs 1 mismatch
    r0 = oracle_mod.compare(out, ref, "f64", 1e-6, 1e-5, 10)
    assert list(r0.report["index"]) == [2, 3, 4]
    # minValueToCheck = 1e-32: elements 0, 1 are not compared (|ref| <= 1e-32): same mismatches,
    # but max_rel no longer sees 1e-40/0 = inf
    r1 = oracle_mod.compare(out, ref, "f64", 1e-6, 1e-5, 10, min_value=1e-32)
    assert list(r1.report["index"]) == [2, 3, 4] and r1.max_rel_err == 0.5 and r0.max_rel_err == np.inf
    # value bound [0, 1]: 0.6 vs 0.5 is ignored (out inside the bound), 3 vs 2 and NaN are not
    r2 = oracle_mod.compare(out, ref, "f64", 1e-6, 1e-5, 10, bounds=(0.0, 1.0))
    assert list(r2.report["index"]) == [2, 4] and r2.max_abs_err == 1.0
    # integers enter the checks as doubles
    a = np.array([5, 9, -3], dtype=np.int32)
    b = np.array([0, 7, -3], dtype=np.int32)
    r3 = oracle_mod.compare(a, b, "i32", 0, 0, 10, min_value=0.5)
    assert list(r3.report["index"]) == [1] and r3.max_abs_err == 2.0


# ------------------------------------------------------- N4: checksum screen
def _checksum_py(b: bytes):
    """Independent pure-Python statement of the checksum definition (arbitrary ints)."""
    M = (1 << 64) - 1

    def fmix(z):
        z ^= z >> 30
        z = (z * 0xBF58476D1CE4E5B9) & M
        z ^= z >> 27
        z = (z * 0x94D049BB133111EB) & M
        return z ^ (z >> 31)

    s = x = 0
    for i in range((len(b) + 7) // 8):
        w = int.from_bytes(b[8 * i: 8 * i + 8].ljust(8, b"\0"), "little")
        h = fmix((w + i * 0x9E3779B97F4A7C15) & M)
        s = (s + h) & M
        x ^= h
    return s, x


@pytest.mark.parametrize("nbytes", [0, 1, 7, 8, 9, 63, 1000, 4099])
def test_checksum_vs_python(oracle_mod, nbytes):
    rng = np.random.default_rng(nbytes)
    b = rng.integers(0, 256, nbytes, dtype=np.uint8)
    assert oracle_mod.checksum(b) == _checksum_py(b.tobytes())


def test_checksum_properties(oracle_mod):
    rng = np.random.default_rng(1)
    a = rng.integers(0, 256, 1 << 16, dtype=np.uint8)
    base = oracle_mod.checksum(a)
    b = a.copy()
    b[12345] ^= 1  # one bit flip changes it
    assert oracle_mod.checksum(b) != base
    w = a.view(np.uint64).copy()
    w[[10, 20]] = w[[20, 10]]  # swapping two words changes it (position-dependent)
    if w[10] != w[20]:
        assert oracle_mod.checksum(w) != base
    assert oracle_mod.checksum(a.copy()) == base


def _splitmix_known():
    rows = []
    for line in open(os.path.join(os.path.dirname(__file__), "golden", "splitmix64_seed0.txt")):
        line = line.split("#", 1)[0].strip()
        if line:
            k, v = line.split()
            rows.append((int(k), int(v, 16)))
    return rows


def test_checksum_known_answer(oracle_mod):
    """Known SplitMix64 outputs pin the finalizer, the word index term and the reductions."""
    known = _splitmix_known()
    words = np.full(len(known), 0x9E3779B97F4A7C15, dtype=np.uint64)
    s, x = oracle_mod.checksum(words)
    assert s == sum(v for _, v in known) % (1 << 64)
    xr = 0
    for _, v in known:
        xr ^= v
    assert x == xr
    for k, v in known:  # the input generator uses the same finalizer
        assert synth.hash64_py(0, k) == v
