"""NEXT row N3 on CPU: region selection (P:163 verificationOptions) and the
report text, through the library's host-only C entry points."""
import numpy as np
import pytest


@pytest.fixture(scope="module")
def av():
    from conftest import build_lib

    build_lib()
    import paper_conf_ipps_leelv14_b200 as av

    return av


def test_paper_example(av):
    opt = "verificationOptions=complement=0,kernels=main_kernel0"  # P:163, verbatim modulo '_'
    assert av.arc_verify_selected(opt, "main_kernel0")
    assert not av.arc_verify_selected(opt, "main_kernel1")


@pytest.mark.parametrize("opt,name,exp", [
    ("complement=1,kernels=main_kernel0", "main_kernel0", False),
    ("complement=1,kernels=main_kernel0", "main_kernel1", True),
    ("complement=0,kernels=a:b:c", "b", True),
    ("complement=0,kernels=a,b,c", "c", True),  # extra comma tokens are names
    ("complement=0,kernels=a:b", "ab", False),
    ("complement=0", "anything", True),  # no list: every region
    ("complement=1", "anything", True),
    ("kernels=x, complement=1", "x", False),
    ("", "x", True),
    ("foo=bar,kernels=x", "x", True),  # other OpenARC options are ignored
])
def test_selection(av, opt, name, exp):
    assert av.arc_verify_selected(opt, name) == exp


def test_selection_errors_and_env(av, monkeypatch):
    with pytest.raises(av.ArcVerifyError):
        av.arc_verify_selected("complement=2", "x")
    with pytest.raises(av.ArcVerifyError):
        av.arc_verify_selected("bogus", "x")
    monkeypatch.delenv("verificationOptions", raising=False)
    monkeypatch.delenv("ARC_VERIFICATION_OPTIONS", raising=False)
    assert av.arc_verify_selected(None, "k")
    monkeypatch.setenv("verificationOptions", "complement=0,kernels=k")
    assert av.arc_verify_selected(None, "k") and not av.arc_verify_selected(None, "j")


def test_format_result(av):
    rep = np.zeros(2, dtype=av.REPORT_DTYPE)
    rep[0] = (1, 0x7FC00000, 0x3F800000)  # NaN vs 1
    rep[1] = (6, 0xFF800000, 0x7F800000)  # -Inf vs Inf
    res = av.Result(1048576, 45, float("inf"), float("inf"), 2, rep)
    txt = av.format_result("main_kernel0", "f32", 1e-6, 1e-5, res, max_entries=5)
    lines = txt.strip().split("\n")
    assert lines[0].startswith("[arc_verify] main_kernel0: FAILED -- 45 of 1048576 elements differ")
    assert "abs_tol=1e-06, rel_tol=1e-05" in lines[0] and "max_abs_err=inf" in lines[0]
    assert lines[1] == "  [1] out=nan (0x7fc00000) ref=1 (0x3f800000)"
    assert lines[2] == "  [6] out=-inf (0xff800000) ref=inf (0x7f800000)"
    ok = av.format_result("k", "i32", 0, 0, av.Result(10, 0, 0.0, 0.0, 0, rep[:0]))
    assert ok.startswith("[arc_verify] k: passed -- 0 of 10 elements differ (exact)")
