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


REQUIRED_FLAGS = ("-fmad=false", "-ftz=false", "-prec-div=true", "arch=compute_100a,code=sm_100a")


def shipped_build_ok(info: str) -> bool:
    """The flags the bit-exact contract depends on, no fast
    math, no -D override, and the code's own knobs at their defaults."""
    nvcc = info.split("; knobs:")[0]
    return (all(f in nvcc for f in REQUIRED_FLAGS) and "use_fast_math" not in nvcc
            and "-fmad=true" not in nvcc and " -D" not in nvcc and info.endswith("defaults=1"))


def test_shipped_library_build_flags(lib):
    """Checked on the loaded library itself (arc_verify_build_info), not on a log."""
    info = lib.arc_verify_build_info()
    assert shipped_build_ok(info), info


def test_build_info_check_rejects_variants(lib):
    info = lib.arc_verify_build_info()
    assert not shipped_build_ok(info.replace("-fmad=false", "-fmad=true"))
    assert not shipped_build_ok(info.replace("-ftz=false", "-ftz=true"))
    assert not shipped_build_ok(info.replace("; knobs:", " -DARCV_DIRECT_DYN=65536; knobs:"))
    assert not shipped_build_ok(info.replace("defaults=1", "defaults=0"))
    assert not shipped_build_ok(info.replace("-O3", "-O3 --use_fast_math"))


@pytest.mark.slow
def test_variant_build_reports_itself(lib, tmp_path):
    """A real -D variant build (as tools/ab.py makes) says so in its own build_info,
    and leaves the in-tree build.log alone."""
    import importlib.util
    import subprocess
    import sys

    spec = importlib.util.spec_from_file_location(
        "_arcv_build", os.path.join(ROOT, "paper_conf_ipps_leelv14_b200", "_build.py"))
    b = importlib.util.module_from_spec(spec)
    spec.loader.exec_module(b)
    log = os.path.join(ROOT, "paper_conf_ipps_leelv14_b200", "build.log")
    before = open(log).read() if os.path.exists(log) else None
    so = b.build(out=str(tmp_path / "variant.so"), defines=("-DARCV_DIRECT_DYN=65536",))
    after = open(log).read() if os.path.exists(log) else None
    assert before == after
    code = ("import ctypes,sys; l=ctypes.CDLL(sys.argv[1]); f=l.arc_verify_build_info; "
            "f.restype=ctypes.c_char_p; print(f().decode())")
    info = subprocess.run([sys.executable, "-c", code, so], capture_output=True, text=True, check=True).stdout
    assert "ARCV_DIRECT_DYN=65536" in info and info.strip().endswith("defaults=0")
    assert not shipped_build_ok(info.strip())


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
