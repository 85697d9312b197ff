"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle.

Bar: bit-exact -- mismatch count, n_reported, the bit patterns of max_abs_err /
max_rel_err, and every report entry (index, out bits, ref bits) -- on the same
seeded inputs (synth/), for every dtype, size class, alignment, batching,
host/device placement and shard count.
"""
import os
import struct

import numpy as np
import pytest
import torch

import synth

pytestmark = pytest.mark.gpu

NP = {"f32": np.float32, "f64": np.float64, "i32": np.int32, "i64": np.int64, "u8": np.uint8}
TD = synth.TORCH_DTYPES
TILE_ELEMS = {"f32": 4096, "f64": 2048, "i32": 4096, "i64": 2048, "u8": 16384}
FUZZ_SCALE = int(os.environ.get("ARCV_FUZZ_SCALE", "1"))  # longer seeded fuzz runs on demand


def bits(x: float) -> int:
    return struct.unpack("<Q", struct.pack("<d", x))[0]


def assert_same(g, o, what=""):
    assert g.n == o.n, what
    assert g.n_mismatch == o.n_mismatch, what
    assert g.n_reported == o.n_reported, what
    assert bits(g.max_abs_err) == bits(o.max_abs_err), (what, g.max_abs_err, o.max_abs_err)
    assert bits(g.max_rel_err) == bits(o.max_rel_err), (what, g.max_rel_err, o.max_rel_err)
    rep = g.report
    if isinstance(rep, torch.Tensor):
        rep = rep.cpu().numpy().view(o.report.dtype)[: g.n_reported]
    assert np.array_equal(np.asarray(rep[: g.n_reported]), o.report), what


@pytest.fixture(scope="module")
def av():
    assert torch.cuda.is_available(), "GPU tests need a CUDA device"
    import paper_conf_ipps_leelv14_b200 as av

    av.init(0)
    yield av
    av.finalize()


@pytest.fixture(scope="module")
def orc():
    import oracle

    oracle.build()
    return oracle


def run_both(av, orc, out, ref, dt, at, rt, mr, what=""):
    g = av.compare(out, ref, at, rt, mr)
    o = orc.compare(out.cpu().numpy(), ref.cpu().numpy(), dt, at, rt, mr)
    assert_same(g, o, what)
    return g, o


def random_pair(dt, n, seed, rate=0.01, device="cuda"):
    gen = torch.Generator(device="cpu").manual_seed(seed)
    if dt in ("f32", "f64"):
        ref = (torch.rand(n, generator=gen, dtype=torch.float64) * 4 - 2).to(TD[dt])
        ibits = torch.int32 if dt == "f32" else torch.int64
        k = torch.randint(-90, 90, (n,), generator=gen).to(ibits)
        out = (ref.view(ibits) + k).view(TD[dt])
        m = torch.rand(n, generator=gen) < rate
        out[m] = out[m] * 1.5 + 0.25
    else:
        hi = 255 if dt == "u8" else 1 << 30
        ref = torch.randint(0, hi, (n,), generator=gen).to(TD[dt])
        out = ref.clone()
        m = torch.rand(n, generator=gen) < rate
        out[m] = (out[m] ^ 3) if dt != "u8" else (out[m] ^ 3)
    return out.to(device), ref.to(device)


# ------------------------------------------------------------------ configs
def test_c1(av, orc):
    c1 = synth.C1()
    out, ref = c1.slice()
    g, o = run_both(av, orc, out.cuda(), ref.cuda(), "f32", c1.abs_tol, c1.rel_tol, c1.max_report, "C1")
    assert g.n_mismatch == 45 and list(g.report["index"]) == c1.planted()


@pytest.mark.parametrize("tol", synth.TOL_PAIRS)
def test_special_pairs(av, orc, tol):
    sp = np.array(synth.F32_SPECIAL_BITS, dtype=np.uint32).view(np.float32)
    out = torch.from_numpy(np.repeat(sp, sp.size)).cuda()
    ref = torch.from_numpy(np.tile(sp, sp.size)).cuda()
    run_both(av, orc, out, ref, "f32", tol[0], tol[1], 10 ** 6, f"specials {tol}")
    # the same values widened to fp64 inputs
    run_both(av, orc, out.double(), ref.double(), "f64", tol[0], tol[1], 10 ** 6, f"specials64 {tol}")


def test_subnormal_canary(av, orc):
    """fp32 subnormals must not be flushed by the widening (reading R8)."""
    out = torch.tensor([1.4e-45, 1.1754942e-38, -1.4e-45], dtype=torch.float32).cuda()
    ref = torch.zeros(3, dtype=torch.float32).cuda()
    g, _ = run_both(av, orc, out, ref, "f32", 0.0, 0.0, 8)
    assert g.n_mismatch == 3 and g.max_abs_err == float(np.float32(1.1754942e-38))


@pytest.mark.parametrize("variant", ["A", "B"])
def test_c2(av, orc, variant):
    c2 = synth.C2(variant)
    out, ref = c2.slice(device="cuda")
    g, _ = run_both(av, orc, out, ref, "f32", c2.abs_tol, c2.rel_tol, c2.max_report, f"C2{variant}")
    assert list(g.report["index"]) == c2.planted()


# ----------------------------------------------------- sizes / alignment
def _sizes(dt):
    te = TILE_ELEMS[dt]
    return sorted({0, 1, 2, 7, 31, 33, 255, te - 1, te, te + 1, 3 * te + 17, 148 * 3 * te + 5, (1 << 20) + 1})


@pytest.mark.parametrize("dt", ["f32", "f64", "i32", "i64", "u8"])
def test_sizes_and_misalignment(av, orc, dt):
    for n in _sizes(dt):
        for off in (0, 1, 3) if n < 1 << 16 else (0, 1):
            big_o, big_r = random_pair(dt, n + off + 3, seed=n * 7 + off)
            out, ref = big_o[off:off + n], big_r[off:off + n]  # storage offset -> misaligned windows
            for mr in (0, 1, 64, 10 ** 9):
                run_both(av, orc, out, ref, dt, 1e-6, 1e-5, mr, f"{dt} n={n} off={off} mr={mr}")


@pytest.mark.parametrize("dt", ["f32", "i32", "u8"])
def test_all_mismatch_and_report_limits(av, orc, dt):
    n = 3 * TILE_ELEMS[dt] + 11
    _, ref = random_pair(dt, n, seed=5, rate=0.0)
    out = ref + 1 if dt != "u8" else (ref ^ 1)
    for mr in (1, n - 1, n, n + 5):
        run_both(av, orc, out, ref, dt, 0.0, 0.0, mr, f"all-mismatch {dt} mr={mr}")


@pytest.mark.parametrize("dt", ["i32", "i64"])
def test_integer_extremes(av, orc, dt):
    """|a - b| at the ends of the range (i32: up to 2^32 - 1, exact in the 32-bit
    path; i64: up to 2^64 - 1, rounded to double) -- reading R9."""
    info = np.iinfo(NP[dt])
    lo, hi = int(info.min), int(info.max)
    vals = [lo, lo + 1, -1, 0, 1, hi - 1, hi]
    pairs = [(a, b) for a in vals for b in vals]
    n = 3 * TILE_ELEMS[dt] + 5  # several tiles and a ragged tail; extremes in every tile
    gen = np.random.default_rng(11)
    ref = gen.integers(lo, hi, size=n, dtype=NP[dt], endpoint=True)
    out = ref.copy()
    for t in range(4):
        for k, (a, b) in enumerate(pairs):
            i = min(n - 1, t * TILE_ELEMS[dt] + 3 * k)
            out[i], ref[i] = a, b
    o, r = torch.from_numpy(out).cuda(), torch.from_numpy(ref).cuda()
    for mr in (0, 7, 10 ** 6):
        g, _ = run_both(av, orc, o, r, dt, 0, 0, mr, f"{dt} extremes mr={mr}")
    assert g.max_abs_err == float(hi - lo)


def test_aliasing(av, orc):
    c1 = synth.C1()
    out, _ = c1.slice()
    out = out.cuda()
    g, _ = run_both(av, orc, out, out, "f32", 0.0, 0.0, 100)
    assert g.n_mismatch == 0  # NaN matches itself (rule 2)


def test_device_report(av, orc):
    c1 = synth.C1()
    out, ref = c1.slice()
    out, ref = out.cuda(), ref.cuda()
    rep = torch.zeros(100 * 24, dtype=torch.uint8, device="cuda")
    g = av.compare(out, ref, c1.abs_tol, c1.rel_tol, 100, report=rep)
    o = orc.compare(out.cpu().numpy(), ref.cpu().numpy(), "f32", c1.abs_tol, c1.rel_tol, 100)
    assert_same(g, o)


def test_repeated_calls_are_stable(av, orc):
    c1 = synth.C1()
    out, ref = c1.slice()
    out, ref = out.cuda(), ref.cuda()
    o = orc.compare(out.cpu().numpy(), ref.cpu().numpy(), "f32", 1e-6, 1e-5, 40)
    o2 = orc.compare(out[:5000].cpu().numpy(), ref[:5000].cpu().numpy(), "f32", 1e-6, 1e-5, 3)
    for _ in range(40):
        assert_same(av.compare(out, ref, 1e-6, 1e-5, 40), o)
        assert_same(av.compare(out[:5000], ref[:5000], 1e-6, 1e-5, 3), o2)


# ------------------------------------------------------------------ batch
def _c3_tensors(device="cuda"):
    regs = synth.c3_regions()
    return regs, [(r, *r.slice(device=device)) for r in regs]


def test_c3_batch_matches_oracle_and_singles(av, orc):
    regs, data = _c3_tensors()
    res = av.batch([(o, r, reg.abs_tol, reg.rel_tol, reg.max_report, reg.name) for reg, o, r in data])
    for (reg, o, r), g in zip(data, res):
        exp = orc.compare(o.cpu().numpy(), r.cpu().numpy(), reg.dtype, reg.abs_tol, reg.rel_tol, reg.max_report)
        assert_same(g, exp, reg.name)
        assert list(g.report["index"]) == reg.planted()
        single = av.compare(o, r, reg.abs_tol, reg.rel_tol, reg.max_report)
        assert_same(single, exp, reg.name + " single")
    # the prepared batch (table built once), called repeatedly, gives the same results
    pb = av.prepare_batch([(o, r, reg.abs_tol, reg.rel_tol, reg.max_report, reg.name) for reg, o, r in data])
    for _ in range(3):
        for g, h in zip(pb(), res):
            assert_same(g, h, "prepared batch")


def test_c3_batch_misaligned_packing(av, orc):
    """All twelve regions packed into one byte buffer at odd element offsets."""
    regs, data = _c3_tensors()
    total = sum((o.numel() + 3) * o.element_size() + 64 for _, o, _ in data)
    bo = torch.zeros(total, dtype=torch.uint8, device="cuda")
    br = torch.zeros(total, dtype=torch.uint8, device="cuda")
    views, pos = [], 0
    for k, (reg, o, r) in enumerate(data):
        es = o.element_size()
        pos = (pos + 15) // 16 * 16 + es * (1 + 2 * (k % 3))  # odd element offset from 16B
        nb = o.numel() * es
        bo[pos:pos + nb].copy_(o.view(torch.uint8))
        br[pos:pos + nb].copy_(r.view(torch.uint8))
        views.append((reg, bo[pos:pos + nb].view(o.dtype), br[pos:pos + nb].view(o.dtype)))
        pos += nb
    res = av.batch([(o, r, reg.abs_tol, reg.rel_tol, 7, reg.name) for reg, o, r in views])
    for (reg, o, r), g in zip(views, res):
        exp = orc.compare(o.cpu().numpy(), r.cpu().numpy(), reg.dtype, reg.abs_tol, reg.rel_tol, 7)
        assert_same(g, exp, reg.name)


def test_batch_many_regions_table_path(av, orc):
    """> 16 segments go through the device descriptor table; include empty regions."""
    items, exps = [], []
    for k in range(37):
        dt = ["f32", "f64", "i32", "i64", "u8"][k % 5]
        n = [0, 1, 5000, 40000, 4097][k % 5] + k
        o, r = random_pair(dt, n, seed=100 + k, rate=0.02)
        items.append((o, r, 1e-6, 1e-5, [0, 3, 1000][k % 3]))
        exps.append(orc.compare(o.cpu().numpy(), r.cpu().numpy(), dt, 1e-6, 1e-5, [0, 3, 1000][k % 3]))
    for g, e in zip(av.batch(items), exps):
        assert_same(g, e)
    # the pinned descriptor table is reused call after call (event-ordered, no stream sync)
    pb = av.prepare_batch(items)
    half = av.prepare_batch(items[::2])
    for _ in range(3):
        for g, e in zip(pb(), exps):
            assert_same(g, e, "prepared")
        for g, e in zip(half(), exps[::2]):
            assert_same(g, e, "prepared half")


@pytest.mark.parametrize("buf", ["pinned_large", "pageable"])
def test_batch_sparse_region_next_to_dense(av, orc, buf):
    """A sparse region (10 mismatches) batched with a dense one that overflows the pool
    (> 2048 nonzero tiles -> group path): the sparse region's entries take the direct
    route (pinned caller buffer, or the library's pinned staging for a pageable one) on
    both report paths, and the host applies the same rule."""
    oa, ra = random_pair("f32", 300_000, seed=71, rate=0.0)
    idx = torch.tensor([5, 77, 4096, 9000, 123456, 200001, 250000, 299990, 299998, 299999])
    oa[idx.cuda()] += 1.0
    ob, rb = synth.C5(1 << 24).slice(device="cuda")  # 4096 nonzero tiles
    cap = 100_000  # > the 2^16 small-pinned limit: the sparse rule decides
    if buf == "pinned_large":
        rep_a = torch.empty(24 * cap, dtype=torch.uint8, pin_memory=True).numpy().view(av.REPORT_DTYPE)
    else:
        rep_a = np.zeros(cap, dtype=av.REPORT_DTYPE)
    pb = av.prepare_batch([(oa, ra, 1e-6, 1e-5, cap), (ob, rb, 0, 0, 5000)], report_buffers=[rep_a, None])
    ea = orc.compare(oa.cpu().numpy(), ra.cpu().numpy(), "f32", 1e-6, 1e-5, cap)
    eb = orc.compare(ob.cpu().numpy(), rb.cpu().numpy(), "i32", 0, 0, 5000)
    for _ in range(2):
        rep_a[:] = np.zeros(1, dtype=av.REPORT_DTYPE)  # stale-free check
        ga, gb = pb()
        assert_same(ga, ea, f"sparse {buf}")
        assert_same(gb, eb, "dense")
    # and the same region alone (pool path)
    g = av.compare(oa, ra, 1e-6, 1e-5, cap, report=rep_a)
    assert_same(g, ea, f"alone {buf}")


@pytest.mark.parametrize("buf", ["pinned_small", "pinned_large", "pageable"])
def test_report_visibility_stress(av, orc, buf):
    """The host reads report entries written over PCIe by many CTAs, ordered only by the
    last CTA's cumulative system fence before the completion word: poison the buffer before
    every call and check every entry, over many back-to-back calls alternating two inputs."""
    cases = []
    for seed in (11, 12):
        reg = synth.configs.Region("S", "f64", 1 << 22, 3000 + seed, 1e-6, 1e-5, 1 << 20, "f64",
                                   n_inject=300 + seed, n_nan=2)
        o, r = reg.slice(device="cuda")
        e = orc.compare(o.cpu().numpy(), r.cpu().numpy(), "f64", 1e-6, 1e-5, 5000)
        cases.append((o, r, e))
    cap = {"pinned_small": 5000, "pinned_large": 1 << 17, "pageable": 5000}[buf]
    if buf == "pageable":
        rep = np.zeros(cap, dtype=av.REPORT_DTYPE)
    else:
        rep = torch.empty(24 * cap, dtype=torch.uint8, pin_memory=True).numpy().view(av.REPORT_DTYPE)
    calls = [av.prepare(o, r, 1e-6, 1e-5, 5000, report=rep) for o, r, _ in cases]
    poison = np.frombuffer(b"\xff" * 24, dtype=av.REPORT_DTYPE)[0]
    for it in range(200):
        k = it & 1
        rep[:] = poison
        g = calls[k]()
        e = cases[k][2]
        assert g.n_mismatch == e.n_mismatch and g.n_reported == e.n_reported, it
        assert np.array_equal(rep[: g.n_reported], e.report), (buf, it)


def test_randomized_fuzz(av, orc):
    """Seeded fuzz: dtype, length, mismatch density (around the 2048-tile pool boundary and
    dense), element offset, max_report and report-buffer kind drawn at random; every call
    bit-exact against the oracle."""
    rng = np.random.default_rng(20141)
    pinned = torch.empty(24 * 70000, dtype=torch.uint8, pin_memory=True).numpy().view(av.REPORT_DTYPE)
    dev_rep = torch.empty(24 * 70000, dtype=torch.uint8, device="cuda")
    for it in range(60 * FUZZ_SCALE):
        dt = ["f32", "f64", "i32", "i64", "u8"][int(rng.integers(5))]
        te = TILE_ELEMS[dt]
        n = int(rng.integers(1, 3000)) * te // 2 + int(rng.integers(0, te))
        off = int(rng.integers(0, 3))
        rate = float(rng.choice([0.0, 1e-5, 3e-4, 1e-3, 0.05, 0.5]))
        o, r = random_pair(dt, n + off, seed=5000 + it, rate=rate)
        o, r = o[off:], r[off:]
        mr = int(rng.choice([0, 1, 100, 4096, 60000]))
        kind = int(rng.integers(3))
        rep = (None, pinned, dev_rep)[kind]
        e = orc.compare(o.cpu().numpy(), r.cpu().numpy(), dt, 1e-6, 1e-5, mr)
        for rep_call in range(2):
            g = av.compare(o, r, 1e-6, 1e-5, mr, report=rep)
            assert_same(g, e, f"it={it} dt={dt} n={n} off={off} rate={rate} mr={mr} kind={kind} call={rep_call}")


def test_randomized_fuzz_batch_and_host(av, orc):
    """Seeded fuzz over batches (1-20 random regions, mixed dtypes and densities, one grid)
    and host-resident inputs (pinned out/ref streamed in chunks: per-chunk report bases)."""
    rng = np.random.default_rng(20142)
    for it in range(25 * FUZZ_SCALE):
        regs, exps = [], []
        for k in range(int(rng.integers(1, 21))):
            dt = ["f32", "f64", "i32", "i64", "u8"][int(rng.integers(5))]
            n = int(rng.integers(0, 200_000))
            rate = float(rng.choice([0.0, 1e-4, 0.01, 0.3]))
            o, r = random_pair(dt, n, seed=7000 + 50 * it + k, rate=rate)
            mr = int(rng.choice([0, 3, 500, 100000]))
            regs.append((o, r, 1e-6, 1e-5, mr))
            exps.append(orc.compare(o.cpu().numpy(), r.cpu().numpy(), dt, 1e-6, 1e-5, mr))
        for g, e in zip(av.batch(regs), exps):
            assert_same(g, e, f"batch it={it}")
    for it in range(8):
        dt = ["f32", "f64", "i32"][it % 3]
        n = int(rng.integers(1, 40)) * (1 << 20) // 3 + int(rng.integers(0, 5000))
        o, r = random_pair(dt, n, seed=9000 + it, rate=float(rng.choice([1e-6, 1e-4, 0.02])))
        mr = int(rng.choice([10, 5000, 1 << 20]))
        e = orc.compare(o.cpu().numpy(), r.cpu().numpy(), dt, 1e-6, 1e-5, mr)
        ho, hr = o.cpu().pin_memory(), r.cpu().pin_memory()
        for a, b, where in ((o, hr, "ref on host"), (ho, hr, "both on host")):
            assert_same(av.compare(a, b, 1e-6, 1e-5, mr), e, f"host it={it} {where} n={n} mr={mr}")


# ----------------------------------------------------------- host inputs
@pytest.mark.parametrize("where", ["ref_pinned", "both_pinned", "ref_pageable"])
def test_host_inputs_streamed(av, orc, where):
    n = 40_000_003  # > 2 chunks of 64 MiB fp32
    c = synth.C4(n)  # fp64 recipe at a smaller n
    out, ref = c.slice(device="cuda")
    o = orc.compare(out.cpu().numpy(), ref.cpu().numpy(), "f64", c.abs_tol, c.rel_tol, 300)
    if where == "ref_pinned":
        a, b = out, ref.cpu().pin_memory()
    elif where == "both_pinned":
        a, b = out.cpu().pin_memory(), ref.cpu().pin_memory()
    else:
        a, b = out, ref.cpu()
    g = av.compare(a, b, c.abs_tol, c.rel_tol, 300)
    assert_same(g, o, where)


# ------------------------------------------------------------ stage variants
@pytest.mark.parametrize("stages,ctas,flags,fused", [(2, 0, 0, 1), (4, 0, 0, 1), (6, 0, 0, 1), (3, 1, 0, 1),
                                                     (3, 0, 8, 1), (3, 0, 0, 0), (4, 1, 0, 0)])
def test_launch_geometry_invariance(orc, stages, ctas, flags, fused):
    """Stage counts, CTAs per SM, (flags=8) stream-sync instead of the completion word, and
    (fused=0, or 2 stages) the report phase as its own launch (K2) instead of K1's tail."""
    import paper_conf_ipps_leelv14_b200 as av

    av.finalize()
    os.environ["ARCV_STAGES"], os.environ["ARCV_CTAS_PER_SM"] = str(stages), str(ctas)
    os.environ["ARCV_FLAGS"], os.environ["ARCV_FUSED"] = str(flags), str(fused)
    try:
        av.init(0)
        c1 = synth.C1()
        out, ref = c1.slice()
        run_both(av, orc, out.cuda(), ref.cuda(), "f32", 1e-6, 1e-5, 30, f"stages={stages}")
        o5, r5 = synth.C5(1 << 22).slice(device="cuda")
        run_both(av, orc, o5, r5, "i32", 0, 0, 5000, f"c5 stages={stages}")
        c4 = synth.C4(1 << 22)
        o4, r4 = c4.slice(device="cuda")
        run_both(av, orc, o4, r4, "f64", 1e-6, 1e-5, 300, f"c4 stages={stages} flags={flags}")
        run_both(av, orc, o4.cpu().pin_memory(), r4, "f64", 1e-6, 1e-5, 300, f"c4 host flags={flags}")
    finally:
        av.finalize()
        del os.environ["ARCV_STAGES"], os.environ["ARCV_CTAS_PER_SM"], os.environ["ARCV_FLAGS"]
        del os.environ["ARCV_FUSED"]
        av.init(0)


@pytest.mark.parametrize("n_tiles", [1, 295, 296, 297, 2047, 2048, 2049, 2050, 2056])
def test_pool_capacity_boundary(av, orc, n_tiles):
    """One mismatch in each of `n_tiles` distinct tiles: up to 2048 nonzero tiles the report
    phase takes the pool path (several entries per CTA beyond 296), from 2049 the group path."""
    te = TILE_ELEMS["f32"]
    n = 4096 * te + 777  # ragged tail tile
    gen = torch.Generator(device="cpu").manual_seed(7000 + n_tiles)
    ref = (torch.rand(n, generator=gen, dtype=torch.float64) + 0.5).to(torch.float32)
    out = ref.clone()
    tiles = torch.randperm(4097, generator=gen)[:n_tiles]
    pos = torch.randint(0, 777, (n_tiles,), generator=gen)  # valid in the tail tile too
    idx = tiles * te + pos
    out[idx] = out[idx] + 1.0
    out, ref = out.cuda(), ref.cuda()
    for mr in (1, n_tiles // 2 + 1, n_tiles, 1 << 20):
        run_both(av, orc, out, ref, "f32", 1e-6, 1e-5, mr, f"tiles={n_tiles} mr={mr}")
    if n_tiles >= 2048:
        # the overflow decision races between the CTAs that finish the 2048th and
        # later nonzero tiles: repeat (a tile left out of a "full" pool must push
        # the count past 2048, or the pool path would run one tile short)
        e = orc.compare(out.cpu().numpy(), ref.cpu().numpy(), "f32", 1e-6, 1e-5, 1 << 20)
        for it in range(40):
            assert_same(av.compare(out, ref, 1e-6, 1e-5, 1 << 20), e, f"tiles={n_tiles} repeat {it}")


# --------------------------------------------------------------- full sizes
def test_c4_full_size(av, orc):
    c4 = synth.C4()
    out, ref = c4.slice(device="cuda")
    g = av.compare(out, ref, c4.abs_tol, c4.rel_tol, c4.max_report)
    o = orc.compare(out.cpu().numpy(), ref.cpu().numpy(), "f64", c4.abs_tol, c4.rel_tol, c4.max_report)
    assert_same(g, o, "C4")
    assert g.n_mismatch == 516 and list(g.report["index"]) == c4.planted()


def test_c5_full_size(av, orc):
    """C5 at its full size (2^30 int32, 8 GiB read) against the oracle over the WHOLE
    arrays (all host cores: compare_threads), plus the generator's closed form."""
    c5 = synth.C5()
    out, ref = c5.slice(device="cuda")
    for rep in (None, torch.empty(24 * c5.max_report, dtype=torch.uint8, device="cuda")):
        g = av.compare(out, ref, 0, 0, c5.max_report, report=rep)
        # closed form: every odd index mismatches by exactly 1
        assert g.n_mismatch == 1 << 29 and g.n_reported == 1 << 20
        assert g.max_abs_err == 1.0 and g.max_rel_err == 0.0
        if rep is None:
            first = g
    o = orc.compare_threads(out.cpu().numpy(), ref.cpu().numpy(), "i32", 0, 0, c5.max_report)
    assert_same(first, o, "C5 full")
    assert_same(g, o, "C5 full, device report")
    assert np.array_equal(o.report["index"], np.arange(1, 1 << 21, 2, dtype=np.uint64))


def test_index_beyond_2_pow_32(av, orc):
    n = (1 << 32) + 4099
    ref = torch.zeros(n, dtype=torch.uint8, device="cuda")
    out = torch.zeros(n, dtype=torch.uint8, device="cuda")
    planted = [5, (1 << 31) + 1, (1 << 32) - 1, 1 << 32, n - 1]
    for i in planted:
        out[i] = 9
    g = av.compare(out, ref, 0, 0, 100)
    assert g.n_mismatch == len(planted) and list(g.report["index"]) == planted
    assert g.max_abs_err == 9.0
    tail = n - (1 << 32) + 10
    o = orc.compare(out[-tail:].cpu().numpy(), ref[-tail:].cpu().numpy(), "u8", 0, 0, 100)
    assert [int(i) + n - tail for i in o.report["index"]] == planted[2:]


# ------------------------------------------------------- sharded loopback
def _loopback(av, out, ref, dt, at, rt, mr, cuts, K):
    p = len(cuts) - 1
    stride = av.arc_verify_packet_bytes(K)
    need = [av.arc_verify_packet_bytes(max(K, min(mr, b - a))) for a, b in zip(cuts[:-1], cuts[1:])]
    gathered = torch.zeros(stride * p, dtype=torch.uint8, device="cuda")
    code = av.DTYPE_CODES[dt]
    for r, (a, b) in enumerate(zip(cuts[:-1], cuts[1:])):
        pk = torch.zeros(need[r], dtype=torch.uint8, device="cuda")
        o, f = out[a:b], ref[a:b]
        av.arc_verify_shard_local(o.data_ptr() if b > a else 0, f.data_ptr() if b > a else 0, b - a, code,
                                  at, rt, mr, pk.data_ptr(), K)
        gathered[r * stride:(r + 1) * stride].copy_(pk[:stride])
    res = av.arc_verify_result_t()
    rep = np.zeros(max(mr, 1), dtype=av.REPORT_DTYPE)
    res.report = rep.ctypes.data
    av.arc_verify_shard_merge(gathered.data_ptr(), p, K, mr, res)
    return av.Result(res.n, res.n_mismatch, res.max_abs_err, res.max_rel_err, res.n_reported, rep[: res.n_reported])


@pytest.mark.parametrize("p", [1, 2, 3, 8])
def test_shard_loopback_matches_unsharded(av, orc, p):
    c1 = synth.C1()
    out, ref = c1.slice()
    out, ref = out.cuda(), ref.cuda()
    n = out.numel()
    cuts = [0] + sorted(synth.distinct_indices(7 + p, p - 1, 1, n)) + [n]
    for mr in (0, 10, 45, 200):
        exp = orc.compare(out.cpu().numpy(), ref.cpu().numpy(), "f32", 1e-6, 1e-5, mr)
        g = _loopback(av, out, ref, "f32", 1e-6, 1e-5, mr, cuts, K=max(mr, 1))
        assert_same(g, exp, f"p={p} mr={mr}")


def test_shard_loopback_int_worst_case(av, orc):
    c5 = synth.C5(1 << 24)
    out, ref = c5.slice(device="cuda")
    n = out.numel()
    cuts = [k * n // 8 for k in range(9)]
    mr = 1 << 20
    exp = orc.compare(out.cpu().numpy(), ref.cpu().numpy(), "i32", 0, 0, mr)
    g = _loopback(av, out, ref, "i32", 0, 0, mr, cuts, K=mr)
    assert_same(g, exp, "c5 loopback")


# ------------------------------------------------------------ bad arguments
def test_invalid_arguments(av):
    x = torch.zeros(16, device="cuda")
    with pytest.raises(av.ArcVerifyError, match="invalid argument"):
        av.compare(x, x, -1.0, 0.0, 4)
    with pytest.raises(av.ArcVerifyError, match="invalid argument"):
        av.compare(x, x, 0.0, float("nan"), 4)
    xb = torch.zeros(64, dtype=torch.uint8, device="cuda")
    mis = xb[1:33].view(torch.uint8)
    r = av.arc_verify_result_t()
    st = av._lib.arc_verify_compare(mis.data_ptr(), mis.data_ptr(), 8, av.ARC_F32, 0.0, 0.0, 0,
                                    __import__("ctypes").byref(r))
    assert st == av.ARC_E_INVAL  # fp32 pointer not 4-byte aligned
    st = av._lib.arc_verify_compare(None, None, 8, av.ARC_F32, 0.0, 0.0, 0, __import__("ctypes").byref(r))
    assert st == av.ARC_E_INVAL


# ------------------------------------------------ pre-filter boundary stress
def _boundary(rng, n, dt):
    if dt == "f32":
        ref = rng.uniform(-4, 4, n).astype(np.float32)
        ref[::17] = 0
        k = rng.integers(-140, 140, n).astype(np.int64)
        out = (ref.view(np.int32).astype(np.int64) + np.where(ref == 0, 0, k)).astype(np.int32).view(np.float32).copy()
        out[::23] = rng.uniform(-2e-6, 2e-6, out[::23].size).astype(np.float32)
    else:
        ref = rng.uniform(-4, 4, n)
        ref[::17] = 0
        k = rng.integers(-1 << 34, 1 << 34, n)
        out = (ref.view(np.int64) + np.where(ref == 0, 0, k)).view(np.float64).copy()
        out[::23] = rng.uniform(-2e-6, 2e-6, out[::23].size)
    return out, ref


@pytest.mark.parametrize("dt", ["f32", "f64"])
@pytest.mark.parametrize("tol", [(1e-6, 1e-5), (0.0, 1e-5), (1e-6, 0.0), (0.0, 0.0), (0.5, 0.3), (0.0, 3.0)])
def test_prefilter_boundaries(av, orc, dt, tol):
    rng = np.random.default_rng(11)
    out, ref = _boundary(rng, 3_000_017, dt)
    run_both(av, orc, torch.from_numpy(out).cuda(), torch.from_numpy(ref).cuda(), dt, tol[0], tol[1], 5000,
             f"boundary {dt} {tol}")


def test_prefilter_ulp_sweep(av, orc):
    """Every fp32 out within +-160 ulps of a spread of refs, at several tolerances."""
    refs = np.array([1.0, 0.75, -3.0, 1e-3, 12345.0, 1e-38, 3e38, 2.0 ** -126], dtype=np.float32)
    k = np.arange(-160, 161)
    outs, rs = [], []
    for y in refs:
        outs.append((np.int64(np.float32(y).view(np.int32)) + k).astype(np.int32).view(np.float32))
        rs.append(np.full(k.size, y, dtype=np.float32))
    out = np.tile(np.concatenate(outs), 50)
    ref = np.tile(np.concatenate(rs), 50)
    for at, rt in [(1e-6, 1e-5), (0.0, 1e-5), (0.0, 1.2e-7), (1e-40, 0.0)]:
        run_both(av, orc, torch.from_numpy(out).cuda(), torch.from_numpy(ref).cuda(), "f32", at, rt, 100000,
                 f"ulp sweep {at} {rt}")


@pytest.mark.parametrize("mr", [100, (1 << 16) + 1])
def test_pinned_report(av, orc, mr):
    """Pinned host report buffers: small ones are written by the kernel over PCIe,
    large ones staged; both must equal the oracle."""
    o5, r5 = synth.C5(1 << 20).slice(device="cuda")
    rep = torch.empty(24 * mr, dtype=torch.uint8, pin_memory=True).numpy().view(av.REPORT_DTYPE)
    g = av.compare(o5, r5, 0, 0, mr, report=rep)
    o = orc.compare(o5.cpu().numpy(), r5.cpu().numpy(), "i32", 0, 0, mr)
    assert_same(g, o, f"pinned mr={mr}")


@pytest.mark.parametrize("n_mis", [0, 1, 4095, 4096, 4097, 20000])
def test_pinned_report_sparse_direct(av, orc, n_mis):
    """A large pinned host report (capacity > 2^16) with <= 4096 mismatches is written by K2
    over PCIe (no D2H copy); with more it goes through HBM staging.  Both sides of the 4096
    boundary, a stale buffer (pre-filled with garbage) and a batch with two such regions."""
    n = 1 << 22
    gen = torch.Generator().manual_seed(n_mis + 7)
    ref = torch.randint(-(1 << 30), 1 << 30, (n,), generator=gen, dtype=torch.int32)
    out = ref.clone()
    idx = torch.randperm(n, generator=gen)[:n_mis]
    out[idx] ^= 5
    mr = 1 << 20
    rep = torch.empty(24 * mr, dtype=torch.uint8, pin_memory=True).numpy().view(av.REPORT_DTYPE)
    rep.view(np.uint8)[:] = 0xA5
    o = orc.compare(out.numpy(), ref.numpy(), "i32", 0, 0, mr)
    for _ in range(2):
        g = av.compare(out.cuda(), ref.cuda(), 0, 0, mr, report=rep)
        assert_same(g, o, f"sparse direct n_mis={n_mis}")
    if n_mis in (1, 4097):
        res = av.batch([(out.cuda(), ref.cuda(), 0, 0, mr), (ref.cuda(), out.cuda(), 0, 0, mr)])
        o2 = orc.compare(ref.numpy(), out.numpy(), "i32", 0, 0, mr)
        assert_same(res[0], o, "batch 0")
        assert_same(res[1], o2, "batch 1")


@pytest.mark.parametrize("n", [1, 15, 16, 17, 16384 * 3 + 5, (1 << 22) + 3])
def test_u8_simd_path(av, orc, n):
    gen = torch.Generator().manual_seed(n)
    ref = torch.randint(0, 256, (n + 5,), generator=gen, dtype=torch.int32).to(torch.uint8)
    out = ref.clone()
    m = torch.rand(n + 5, generator=gen) < 0.003
    out[m] = torch.randint(0, 256, (int(m.sum()),), generator=gen, dtype=torch.int32).to(torch.uint8)
    for off in (0, 3):
        o, r = out.cuda()[off:off + n], ref.cuda()[off:off + n]
        run_both(av, orc, o, r, "u8", 0, 0, 1000, f"u8 n={n} off={off}")


def test_collective_path_one_rank_nccl():
    """The sharded/collective code path (NCCL all-gather + merge kernel + broadcast)
    on a 1-rank communicator, in its own process (one library context per process)."""
    import subprocess
    import sys

    script = os.path.join(os.path.dirname(__file__), "_nccl_one_rank.py")
    res = subprocess.run([sys.executable, script], capture_output=True, text=True, timeout=600)
    assert res.returncode == 0, res.stdout[-3000:] + res.stderr[-3000:]
    assert "NCCL-ONE-RANK-OK" in res.stdout


def test_host_streamed_dense_group_path(av, orc):
    """Host-resident inputs with dense mismatches: chunked launches whose nonzero
    tiles overflow K2's pool, so the group path runs with a per-chunk base."""
    c5 = synth.C5(1 << 25)
    out, ref = c5.slice()
    mr = (1 << 24) + 7  # reaches into the second chunk
    rep = np.zeros(mr, dtype=av.REPORT_DTYPE)
    g = av.compare(out.pin_memory(), ref, 0, 0, mr, report=rep)
    o = orc.compare(out.numpy(), ref.numpy(), "i32", 0, 0, mr)
    assert_same(g, o, "host streamed dense")


def test_pool_and_group_paths_alternate(av, orc):
    """K2's sparse pool path and dense group path interleaved (shared counters,
    grid-barrier bookkeeping) stay correct call after call."""
    c1 = synth.C1()
    o1, r1 = c1.slice()
    o5, r5 = synth.C5(1 << 24).slice()  # 4096 nonzero tiles > pool capacity
    e1 = orc.compare(o1.numpy(), r1.numpy(), "f32", 1e-6, 1e-5, 100)
    e5 = orc.compare(o5.numpy(), r5.numpy(), "i32", 0, 0, 5000)
    o1, r1, o5, r5 = o1.cuda(), r1.cuda(), o5.cuda(), r5.cuda()
    for _ in range(6):
        assert_same(av.compare(o1, r1, 1e-6, 1e-5, 100), e1, "pool")
        assert_same(av.compare(o5, r5, 0, 0, 5000), e5, "group")
        assert_same(av.compare(o1, r1, 1e-6, 1e-5, 100), e1, "pool again")


# ---------------------------------------------- N2: minValueToCheck / bounds
CHECKS = [(1e-32, None), (0.5, None), (None, (-0.25, 0.25)), (1e-3, (0.0, 1.0)), (0.0, (-np.inf, np.inf))]


@pytest.mark.parametrize("dt", ["f32", "f64"])
@pytest.mark.parametrize("mv,bounds", CHECKS)
def test_checks_float(av, orc, dt, mv, bounds):
    rng = np.random.default_rng(5)
    out, ref = _boundary(rng, 1_000_003, dt)
    sp = np.array(synth.F32_SPECIAL_BITS, dtype=np.uint32).view(np.float32).astype(NP[dt])
    out = np.concatenate([out, np.repeat(sp, sp.size)])
    ref = np.concatenate([ref, np.tile(sp, sp.size)])
    o, r = torch.from_numpy(out).cuda(), torch.from_numpy(ref).cuda()
    g = av.compare(o, r, 1e-6, 1e-5, 4000, min_value=mv, bounds=bounds)
    e = orc.compare(out, ref, dt, 1e-6, 1e-5, 4000, min_value=mv, bounds=bounds)
    assert_same(g, e, f"checks {dt} {mv} {bounds}")


@pytest.mark.parametrize("dt", ["i32", "i64", "u8"])
def test_checks_int(av, orc, dt):
    o, r = random_pair(dt, 300_017, seed=9, rate=0.05)
    for mv, bounds in [(3.0, None), (None, (0.0, 100.0)), (200.0, (10.0, 1e9))]:
        g = av.compare(o, r, 0, 0, 1000, min_value=mv, bounds=bounds)
        e = orc.compare(o.cpu().numpy(), r.cpu().numpy(), dt, 0, 0, 1000, min_value=mv, bounds=bounds)
        assert_same(g, e, f"checks {dt} {mv} {bounds}")


def test_checks_batch_and_streamed(av, orc):
    c1 = synth.C1()
    o, r = c1.slice()
    ck = av.make_check(min_value=0.25, bounds=(-0.6, -0.4))
    res = av.batch([(o.cuda(), r.cuda(), 1e-6, 1e-5, 100, "a", ck), (o.cuda(), r.cuda(), 1e-6, 1e-5, 100, "b")])
    e_ck = orc.compare(o.numpy(), r.numpy(), "f32", 1e-6, 1e-5, 100, min_value=0.25, bounds=(-0.6, -0.4))
    e = orc.compare(o.numpy(), r.numpy(), "f32", 1e-6, 1e-5, 100)
    assert_same(res[0], e_ck, "batch checked")
    assert_same(res[1], e, "batch plain")
    g = av.compare(o.pin_memory(), r, 1e-6, 1e-5, 100, min_value=0.25, bounds=(-0.6, -0.4))
    assert_same(g, e_ck, "host streamed checked")


# ------------------------------------------------------------- N4: checksum
@pytest.mark.parametrize("nbytes", [0, 1, 7, 8, 15, 16, 17, 4096 * 16 + 9, (1 << 24) + 5])
@pytest.mark.parametrize("off", [0, 1, 8, 13])
def test_checksum_vs_oracle(av, orc, nbytes, off):
    gen = torch.Generator().manual_seed(nbytes + off)
    b = torch.randint(0, 256, (nbytes + off + 8,), generator=gen, dtype=torch.int32).to(torch.uint8)
    d = b.cuda()[off:off + nbytes]
    assert av.checksum(d) == orc.checksum(b[off:off + nbytes].numpy())


def test_checksum_screens_c4(av, orc):
    c4 = synth.C4(1 << 26)
    out, ref = c4.slice(device="cuda")
    assert av.checksum(ref) == orc.checksum(ref.cpu().numpy())
    assert av.checksum(out) != av.checksum(ref)  # noisy output differs
    assert av.checksum(ref.clone()) == av.checksum(ref)


# ------------------------------------------------------ N3: selected batch
def test_batch_selected_paper_options(av, orc):
    regs, data = _c3_tensors()
    items = [(o, r, reg.abs_tol, reg.rel_tol, reg.max_report, reg.name) for reg, o, r in data]
    res = av.batch(items, options="verificationOptions=complement=0,kernels=CG:SPMUL")
    for (reg, o, r), g in zip(data, res):
        if reg.name in ("CG", "SPMUL"):
            e = orc.compare(o.cpu().numpy(), r.cpu().numpy(), reg.dtype, reg.abs_tol, reg.rel_tol, reg.max_report)
            assert_same(g, e, reg.name)
        else:
            assert (g.n, g.n_mismatch, g.n_reported) == (0, 0, 0)
    res = av.batch(items, options="complement=1,kernels=JACOBI")
    for (reg, o, r), g in zip(data, res):
        assert (g.n == 0) == (reg.name == "JACOBI")
    txt = av.format_result("SPMUL", "f32", 1e-6, 1e-5, res[[reg.name for reg, _, _ in data].index("SPMUL")])
    assert txt.startswith("[arc_verify] SPMUL: FAILED")


def test_prepared_call(av, orc):
    c1 = synth.C1()
    o, r = c1.slice()
    e = orc.compare(o.numpy(), r.numpy(), "f32", 1e-6, 1e-5, 60)
    o, r = o.cuda(), r.cuda()
    call = av.prepare(o, r, 1e-6, 1e-5, 60)
    for _ in range(5):
        assert_same(call(), e, "prepared")
    e2 = orc.compare(o.cpu().numpy(), r.cpu().numpy(), "f32", 1e-6, 1e-5, 60, min_value=0.25, bounds=(-0.6, -0.4))
    assert_same(av.prepare(o, r, 1e-6, 1e-5, 60, min_value=0.25, bounds=(-0.6, -0.4))(), e2, "prepared checks")


def test_f32_index_beyond_2_pow_32(av):
    """fp32 arrays of more than 2^32 elements: 64-bit indices through tiles, counts and report."""
    n = (1 << 32) + 1000
    ref = torch.zeros(n, dtype=torch.float32, device="cuda")
    out = torch.zeros(n, dtype=torch.float32, device="cuda")
    planted = [3, (1 << 32) - 2, (1 << 32) + 1, n - 1]
    for i in planted:
        out[i] = 1.0
    g = av.compare(out, ref, 1e-6, 1e-5, 10)
    assert g.n_mismatch == len(planted) and list(g.report["index"]) == planted
    assert g.max_abs_err == 1.0 and g.max_rel_err == float("inf")
    del out, ref
    torch.cuda.empty_cache()


def test_env_flags_cannot_disable_the_predicate():
    """ARCV_FLAGS is a diagnostic knob: only bits 1 and 8 are honoured.  Bit 2 is the
    internal read-probe flag (predicate off); from the environment it must not turn
    every compare into '0 mismatches, ARC_OK'."""
    import subprocess
    import sys

    code = ("import sys; sys.path.insert(0, %r); import synth, paper_conf_ipps_leelv14_b200 as av; "
            "c1 = synth.C1(); o, r = c1.slice(device='cuda'); av.init(0); "
            "g = av.compare(o, r, c1.abs_tol, c1.rel_tol, 100); print('COUNT', g.n_mismatch)"
            % os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    for flags in ("2", "10", "3", "15"):
        env = dict(os.environ, ARCV_FLAGS=flags)
        res = subprocess.run([sys.executable, "-c", code], capture_output=True, text=True, timeout=300, env=env)
        assert res.returncode == 0, res.stderr[-2000:]
        assert "COUNT 45" in res.stdout, (flags, res.stdout)


@pytest.mark.parametrize("dt,n_dense,mr,buf,off", [
    ("f32", 2, 1 << 20, "pinned", 0),      # C2B-like: 2 dense tiles, staged coalesced direct writes
    ("f32", 2, 1 << 20, "pageable", 1),    # library pinned staging, misaligned arrays
    ("f32", 2, 5000, "pinned", 0),         # truncation inside the second tile
    ("f64", 20, 1 << 20, "pinned", 0),     # 40960 entries, pool path, direct
    ("f64", 20, 1 << 20, "pageable", 0),   # > the 2^16 pageable staging: HBM staging + D2H
    ("i32", 100, 1 << 20, "pinned", 3),    # 409600 > 2^18 entries: HBM staging + D2H
    ("i32", 100, 7777, "pinned", 0),       # truncated far below: direct
    ("u8", 3, 1 << 20, "pinned", 5),       # u8 tiles (16384 elements), several staging rounds
    ("f32", 2, 1 << 20, "device", 0),      # device report: plain scattered stores
    ("f32", 1, 1 << 20, "pinned", 0),      # one dense tile
])
def test_dense_tiles_direct_route(av, orc, dt, n_dense, mr, buf, off):
    """Few report tiles holding many mismatches (C2B's shape: a wrong loop bound leaves a
    whole row stale): the pool path writes a dense tile's entries through shared memory as
    coalesced words (in rounds of 1024 entries) -- into the caller's pinned buffer (or the
    library's pinned staging) when direct_route() allows, else into HBM staging followed by
    one D2H copy.  Every combination bit-exact against the oracle."""
    te = TILE_ELEMS[dt]
    n = te * (n_dense * 3 + 5) + 123
    out, ref = random_pair(dt, n + off, seed=4242 + n_dense, rate=0.0)
    out, ref = out[off:], ref[off:]
    for k in range(n_dense):  # every third tile fully mismatching (plus a partial tail)
        t0 = (3 * k + 1) * te
        if dt in ("f32", "f64"):
            out[t0:t0 + te] = ref[t0:t0 + te] * 1.5 + 0.25
        else:
            out[t0:t0 + te] = ref[t0:t0 + te] ^ 1
    if buf == "pinned":
        rep = torch.empty(24 * mr, dtype=torch.uint8, pin_memory=True).numpy().view(av.REPORT_DTYPE)
        rep.view(np.uint8)[:] = 0xA5
    elif buf == "pageable":
        rep = np.full(mr, 0, dtype=av.REPORT_DTYPE)
    else:
        rep = torch.empty(24 * mr, dtype=torch.uint8, device="cuda")
    at, rt = (1e-6, 1e-5) if dt in ("f32", "f64") else (0, 0)
    e = orc.compare(out.cpu().numpy(), ref.cpu().numpy(), dt, at, rt, mr)
    for it in range(3):
        g = av.compare(out, ref, at, rt, mr, report=rep)
        assert_same(g, e, f"{dt} dense={n_dense} mr={mr} {buf} off={off} it={it}")


@pytest.mark.parametrize("kind", ["checks", "batch"])
def test_dense_tiles_checks_and_batches(av, orc, kind):
    """The staged dense-tile route combined with the N2 checks (minValueToCheck and
    value bounds remove some mismatches inside the dense tiles, so K1's counts and the
    report phase's ranks must agree under the checks) and inside a batch (a dense region
    and a sparse one sharing the pool, each with its own pinned report)."""
    te = TILE_ELEMS["f32"]
    n = te * 9 + 77
    out, ref = random_pair("f32", n, seed=777, rate=0.0)
    for t in (2, 6):
        out[t * te:(t + 1) * te] = ref[t * te:(t + 1) * te] * 1.5 + 0.25
    mr = 1 << 20
    pin = lambda cap: torch.empty(24 * cap, dtype=torch.uint8, pin_memory=True).numpy().view(av.REPORT_DTYPE)
    if kind == "checks":
        rep = pin(mr)
        for mv, bounds in ((0.5, None), (None, (-0.2, 0.9)), (0.25, (0.0, 1.0))):
            e = orc.compare(out.cpu().numpy(), ref.cpu().numpy(), "f32", 1e-6, 1e-5, mr, min_value=mv, bounds=bounds)
            g = av.compare(out, ref, 1e-6, 1e-5, mr, report=rep, min_value=mv, bounds=bounds)
            assert_same(g, e, f"dense + checks {mv} {bounds}")
    else:
        o2, r2 = random_pair("f64", 500_000, seed=778, rate=0.0)
        o2[[5, 99_999, 400_000]] += 1.0
        reps = [pin(mr), pin(1000)]
        res = av.prepare_batch([(out, ref, 1e-6, 1e-5, mr), (o2, r2, 1e-6, 1e-5, 1000)], report_buffers=reps)
        e1 = orc.compare(out.cpu().numpy(), ref.cpu().numpy(), "f32", 1e-6, 1e-5, mr)
        e2 = orc.compare(o2.cpu().numpy(), r2.cpu().numpy(), "f64", 1e-6, 1e-5, 1000)
        for it in range(3):
            for b in reps:
                b.view(np.uint8)[:] = 0x5A
            g1, g2 = res()
            assert_same(g1, e1, f"batch dense it={it}")
            assert_same(g2, e2, f"batch sparse it={it}")


# ------------------------------------- clustered mismatches around the pool capacity
@pytest.mark.parametrize("dt", ["f32", "f64", "i32", "i64", "u8"])
@pytest.mark.parametrize("n_mis", [1, 700, 2047, 2048, 2049, 2600])
def test_clustered_mismatches_reuse_tiles(av, orc, dt, n_mis):
    """1 .. 2600 mismatches clustered in six tiles (hundreds per tile: pool path, several
    mismatches per thread, ranks across warps and vectors) plus one in the ragged tail tile,
    every dtype.  Each config alternates with a dense call over the SAME tiles (the report phase
    must leave the per-tile counts clean for the next call), with several truncations, a device
    report, and a two-region batch over overlapping views."""
    te = TILE_ELEMS[dt]
    n = 64 * te + 333
    gen = torch.Generator(device="cpu").manual_seed(9100 + n_mis)
    idx = torch.randperm(6 * te, generator=gen)[:n_mis] + 5 * te  # tiles 5..10: several per tile
    idx[0] = n - 1  # and one in the ragged tail tile
    if dt in ("f32", "f64"):
        ref = (torch.rand(n, generator=gen, dtype=torch.float64) + 0.5).to(TD[dt])
        out = ref.clone()
        out[idx] = out[idx] * 1.5
    else:
        hi = 200 if dt == "u8" else 1 << 30
        ref = torch.randint(0, hi, (n,), generator=gen).to(TD[dt])
        out = ref.clone()
        out[idx] = out[idx] + 7
    dense = ref.clone()
    dense[5 * te: 11 * te] = (dense[5 * te: 11 * te] + 3).to(TD[dt])
    on, rn, dn = out.numpy(), ref.numpy(), dense.numpy()
    out, ref, dense = out.cuda(), ref.cuda(), dense.cuda()
    for mr in (1, n_mis // 2 + 1, 1 << 20):
        e = orc.compare(on, rn, dt, 1e-6, 1e-5, mr)
        ed = orc.compare(dn, rn, dt, 1e-6, 1e-5, mr)
        for it in range(3):
            assert_same(av.compare(out, ref, 1e-6, 1e-5, mr), e, f"{dt} n_mis={n_mis} mr={mr} it={it}")
            assert_same(av.compare(dense, ref, 1e-6, 1e-5, mr), ed, f"{dt} dense mr={mr} it={it}")
    # device report, and a batch of the sparse region with itself (two regions, one capture)
    rep = torch.empty(24 * (1 << 20), dtype=torch.uint8, device="cuda")
    assert_same(av.compare(out, ref, 1e-6, 1e-5, 1 << 20, report=rep), e, f"{dt} device report")
    if n_mis <= 1024:
        gs = av.batch([(out, ref, 1e-6, 1e-5, 1 << 20), (out[te:], ref[te:], 1e-6, 1e-5, 17)])
        assert_same(gs[0], e, f"{dt} batch region 0")
        assert_same(gs[1], orc.compare(on[te:], rn[te:], dt, 1e-6, 1e-5, 17), f"{dt} batch region 1")


def test_generic_and_dtype_specialised_k1_agree(orc):
    """Single-region calls and fp32/fp64/int32 batches run K1s compiled for their dtypes;
    ARCV_DT_SPEC=0 forces the generic K1 (all dtypes).  Both agree with the oracle, every
    dtype, aligned and misaligned, single and batched."""
    import paper_conf_ipps_leelv14_b200 as av

    cases = []
    for k, dt in enumerate(["f32", "f64", "i32", "i64", "u8"]):
        n = 3 * TILE_ELEMS[dt] + 101
        o, r = random_pair(dt, n + 1, 8800 + k, rate=0.002, device="cpu")
        cases.append((dt, o, r, 0))
        cases.append((dt, o, r, 1))  # views one element in: misaligned windows
    expect = [orc.compare(o[off:off + len(o) - 1].numpy(), r[off:off + len(o) - 1].numpy(), dt, 1e-6, 1e-5, 500)
              for dt, o, r, off in cases]
    dev = [(dt, o.cuda(), r.cuda(), off) for dt, o, r, off in cases]
    av.finalize()
    try:
        for spec in ("0", "1"):
            os.environ["ARCV_DT_SPEC"] = spec
            av.init(0)
            views = [(o[off:off + o.numel() - 1], r[off:off + r.numel() - 1]) for _, o, r, off in dev]
            for (dt, _, _, off), (o, r), e in zip(dev, views, expect):
                assert_same(av.compare(o, r, 1e-6, 1e-5, 500), e, f"spec={spec} {dt} off={off}")
            fi = [i for i, (dt, _, _, off) in enumerate(dev) if dt in ("f32", "f64", "i32") and off == 0]
            for i, g in zip(fi, av.batch([(views[i][0], views[i][1], 1e-6, 1e-5, 500) for i in fi])):
                assert_same(g, expect[i], f"spec={spec} batch {dev[i][0]}")
            allb = av.batch([(o, r, 1e-6, 1e-5, 500) for o, r in views])
            for i, g in enumerate(allb):
                assert_same(g, expect[i], f"spec={spec} mixed batch {i}")
            av.finalize()
    finally:
        del os.environ["ARCV_DT_SPEC"]
        av.init(0)
