"""Documentation stays in step with the code (CPU only): every environment knob the
library reads is listed in README.md's knob table, and every K1 translation unit the
build compiles is named in DESIGN.md."""
import glob
import os
import re

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
CSRC = os.path.join(ROOT, "paper_conf_ipps_leelv14_b200", "csrc")


def _read(path):
    with open(path) as f:
        return f.read()


def test_every_environment_knob_is_documented():
    names = set()
    for src in glob.glob(os.path.join(CSRC, "*.cu")):
        text = _read(src)
        names |= set(re.findall(r'env_int\("(ARCV?_[A-Z0-9_]+)"', text))
        names |= set(re.findall(r'getenv\("(ARCV?_[A-Z0-9_]+)"', text))
    assert names, "no knobs found: the pattern no longer matches the sources"
    readme = _read(os.path.join(ROOT, "README.md"))
    missing = sorted(n for n in names if f"`{n}`" not in readme)
    assert not missing, f"knobs read by the library but not in README.md: {missing}"


def test_k1_translation_units_are_described():
    design = _read(os.path.join(ROOT, "DESIGN.md"))
    tus = [os.path.basename(p) for p in glob.glob(os.path.join(CSRC, "arcv_k1_*.cu"))]
    assert tus
    # the per-stage-count TUs (arcv_k1_s<S>.cu) and the dtype-specialised ones (arcv_k1_s3_dt*.cu)
    assert "arcv_k1_s<S>.cu" in design or "arcv_k1_s" in design
    if any(t.startswith("arcv_k1_s3_dt") for t in tus):
        assert "arcv_k1_s3_dt" in design
