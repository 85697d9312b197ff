"""Build libarcverify.so in-tree with nvcc for sm_100a.

Flags that the bit-exact contract depends on:
  -fmad=false      no FMA contraction of abs_tol + rel_tol*|y| (the kernel also
                   uses __dmul_rn/__dadd_rn, so this is belt and braces)
  -ftz=false       fp32 subnormals survive the widening cvt.f64.f32
  -prec-div=true   IEEE division
No --use_fast_math.
"""
from __future__ import annotations

import glob
import json
import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(HERE)
CSRC = os.path.join(HERE, "csrc")
LIB = os.path.join(HERE, "libarcverify.so")
INCLUDE = os.path.join(ROOT, "include")

NVCC_FLAGS = [
    "-gencode", "arch=compute_100a,code=sm_100a",
    "-O3", "-lineinfo", "-std=c++17",
    "-Xcompiler", "-fPIC", "-shared",
    "-fmad=false", "-ftz=false", "-prec-div=true", "-prec-sqrt=true",
    "-Xptxas", "-v",
]


def _nccl_include() -> str:
    try:
        import nvidia.nccl  # the torch wheel's NCCL (2.28.x)

        p = os.path.join(list(nvidia.nccl.__path__)[0], "include")
        if os.path.exists(os.path.join(p, "nccl.h")):
            return p
    except Exception:
        pass
    return "/usr/include"


def sources() -> list[str]:
    return sorted(glob.glob(os.path.join(CSRC, "*.cu")))


def _stale() -> bool:
    if not os.path.exists(LIB):
        return True
    t = os.path.getmtime(LIB)
    deps = sources() + glob.glob(os.path.join(CSRC, "*.h")) + glob.glob(os.path.join(CSRC, "*.cuh")) + glob.glob(os.path.join(INCLUDE, "*.h"))
    return any(os.path.getmtime(d) > t for d in deps)


def build(force: bool = False, verbose: bool = False, out: str | None = None, defines: tuple = ()) -> str:
    """Build the library (in-tree by default).  `out` + `defines` build an A/B
    variant elsewhere (e.g. scratch/var.so with -DARCV_FENCE_SC=1)."""
    target = out or LIB
    if out is None and not force and not _stale():
        return LIB
    nvcc = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
    tmp = target + f".tmp{os.getpid()}"
    # arc_verify_build_info(): the flags and defines this very library was built
    # with, compiled into it through a generated header (tests check the shipped
    # library, not a log a variant build may have overwritten)
    import tempfile

    gen = tempfile.mkdtemp(prefix="arcv_gen_")
    info = " ".join(a for a in NVCC_FLAGS if a not in ("-Xptxas", "-v")) + (" " + " ".join(defines) if defines else "")
    with open(os.path.join(gen, "arcv_build_info.h"), "w") as f:
        f.write("#pragma once\n#define ARCV_BUILD_FLAGS " + json.dumps(info) + "\n")
    # one nvcc per translation unit, in parallel (the K1 stage variants are
    # separate TUs), then one link
    from concurrent.futures import ThreadPoolExecutor

    objdir = tempfile.mkdtemp(prefix="arcv_obj_")
    cflags = [a for a in NVCC_FLAGS if a != "-shared"]
    inc = ["-I", gen, "-I", INCLUDE, "-I", CSRC, "-I", _nccl_include()]

    def compile_one(src):
        obj = os.path.join(objdir, os.path.basename(src) + ".o")
        cmd = [nvcc, *cflags, *defines, *inc, "-c", src, "-o", obj]
        return cmd, obj, subprocess.run(cmd, capture_output=True, text=True)

    with ThreadPoolExecutor(max(1, min(len(sources()), os.cpu_count() or 1))) as ex:
        results = list(ex.map(compile_one, sources()))
    link = [nvcc, "-gencode", "arch=compute_100a,code=sm_100a", "-shared", "-Xcompiler", "-fPIC", "-o", tmp,
            *[o for _, o, _ in results], "-ldl"]
    lres = subprocess.run(link, capture_output=True, text=True) if all(r.returncode == 0 for _, _, r in results) \
        else None
    # the in-tree log belongs to the in-tree library; a variant logs next to itself
    log = os.path.join(HERE, "build.log") if out is None else target + ".build.log"
    text = "".join(" ".join(c) + "\n" + r.stdout + r.stderr for c, _, r in results)
    if lres is not None:
        text += " ".join(link) + "\n" + lres.stdout + lres.stderr
    with open(log, "w") as f:
        f.write(text)
    failed = lres is None or lres.returncode != 0
    if failed:
        sys.stderr.write(text[-20000:])
        raise RuntimeError(f"nvcc failed (see {log})")
    if verbose:
        sys.stderr.write(text)
    os.replace(tmp, target)
    import shutil

    shutil.rmtree(objdir, ignore_errors=True)
    shutil.rmtree(gen, ignore_errors=True)
    return target


if __name__ == "__main__":
    # python _build.py [--force] | python _build.py --variant OUT.so -DNAME=VALUE ...
    if "--variant" in sys.argv:
        i = sys.argv.index("--variant")
        print(build(out=os.path.abspath(sys.argv[i + 1]), defines=tuple(a for a in sys.argv[i + 2:] if a.startswith("-D"))))
    else:
        print(build(force="--force" in sys.argv, verbose=True))
