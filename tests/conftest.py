import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def build_lib():
    """Build libarcverify.so if stale.  _build.py is loaded by path: importing the
    package would try to load the not-yet-built library (it raises without it)."""
    import importlib.util

    spec = importlib.util.spec_from_file_location(
        "_arcv_build", os.path.join(ROOT, "paper_conf_ipps_leelv14_b200", "_build.py"))
    b = importlib.util.module_from_spec(spec)
    spec.loader.exec_module(b)
    return b.build()


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a CUDA device (B200, sm_100a)")
    config.addinivalue_line("markers", "slow: large-size CPU test")


@pytest.fixture(scope="session")
def oracle_mod():
    import oracle

    oracle.build()
    return oracle
