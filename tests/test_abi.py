"""CPU checks of the C-ABI library: it loads, exports every declared symbol,
rejects calls before init, and its host-side merge plan matches the plain
definition.  No compute call is made without a GPU."""
import ctypes
import os
import re

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "arc_verify.h")


@pytest.fixture(scope="module")
def lib():
    from conftest import build_lib

    build_lib()
    import paper_conf_ipps_leelv14_b200 as av

    return av


def declared_symbols():
    src = open(HEADER).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(arc_verify_\w+)\s*\(", src)))


def test_header_declares_the_north_star_calls():
    syms = declared_symbols()
    for s in ("arc_verify_init", "arc_verify_compare", "arc_verify_batch", "arc_verify_finalize"):
        assert s in syms


def test_every_declared_symbol_is_exported(lib):
    so = ctypes.CDLL(lib.LIB_PATH)
    for s in declared_symbols():
        assert hasattr(so, s), s
    assert sorted(lib.EXPORTED) == declared_symbols()


def test_sm100a_cubin_embedded(lib):
    import subprocess

    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "--list-elf", lib.LIB_PATH],
                         capture_output=True, text=True).stdout
    assert "sm_100a" in out


def test_calls_before_init(lib):
    r = lib.arc_verify_result_t()
    st = lib._lib.arc_verify_compare(None, None, 0, 0, 0.0, 0.0, 0, ctypes.byref(r))
    assert st == lib.ARC_E_NOINIT
    assert lib._lib.arc_verify_finalize() == lib.ARC_E_NOINIT
    assert lib._lib.arc_verify_strerror(lib.ARC_E_INVAL) == b"invalid argument"
    assert lib.arc_verify_version() >> 16 == 1
    assert lib.arc_verify_packet_bytes(10) == 32 + 240


def test_merge_plan_host(lib):
    hdrs = [(10, 3, 0x3FF0000000000000, 0), (5, 0, 0, 0), (7, 9, 0x4000000000000000, 0x7FF0000000000000)]
    plan, g = lib.arc_verify_merge_plan(hdrs, 5)
    assert plan == [(0, 0, 3), (10, 3, 0), (15, 3, 2)]
    assert g == (22, 12, 0x4000000000000000, 0x7FF0000000000000)
    plan, g = lib.arc_verify_merge_plan(hdrs, 0)
    assert [p[2] for p in plan] == [0, 0, 0]


def test_kernel_flags_in_build_log(lib):
    log = open(os.path.join(os.path.dirname(lib.LIB_PATH), "build.log")).read()
    first = log.splitlines()[0]
    for flag in ("-fmad=false", "-ftz=false", "-prec-div=true", "arch=compute_100a,code=sm_100a"):
        assert flag in first
    assert "use_fast_math" not in first


def _build_c_example(out_path):
    import subprocess

    cmd = ["gcc", "-std=c99", "-O2", "-Wall", "-Werror", "-I", os.path.join(ROOT, "include"),
           "-I", "/usr/local/cuda/include", os.path.join(ROOT, "examples", "verify_region.c"),
           "-L", os.path.join(ROOT, "paper_conf_ipps_leelv14_b200"), "-larcverify",
           "-L", "/usr/local/cuda/lib64", "-lcudart",
           "-Wl,-rpath," + os.path.join(ROOT, "paper_conf_ipps_leelv14_b200"), "-lm", "-o", out_path]
    return subprocess.run(cmd, capture_output=True, text=True)


def test_c_example_compiles_and_links_as_c99(lib, tmp_path):
    """The ABI is plain C: a C99 program includes the header and links the library."""
    r = _build_c_example(str(tmp_path / "verify_region"))
    assert r.returncode == 0, r.stderr


@pytest.mark.gpu
def test_c_example_runs(lib, tmp_path):
    """The C program verifies a region on the GPU and finds exactly the planted stale row."""
    import subprocess

    exe = str(tmp_path / "verify_region")
    r = _build_c_example(exe)
    assert r.returncode == 0, r.stderr
    p = subprocess.run([exe], capture_output=True, text=True, timeout=120)
    assert p.returncode == 0, p.stdout + p.stderr
    assert "PASS: 998 mismatches" in p.stdout
    assert "main_kernel0" in p.stdout
