import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)
TESTS = os.path.dirname(os.path.abspath(__file__))
if TESTS not in sys.path:
    sys.path.insert(0, TESTS)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a CUDA device (B200); run with -m gpu")
    config.addinivalue_line("markers", "slow: long-running CPU test")


@pytest.fixture(scope="session")
def orc():
    import oracle
    oracle.build()
    return oracle


_cache = {}


def cached_batch(name, **kw):
    """Session cache of generated workloads (generation is deterministic)."""
    from gen import make
    key = (name, tuple(sorted(kw.items())))
    if key not in _cache:
        _cache[key] = make(name, **kw)
    return _cache[key]


@pytest.fixture(scope="session", autouse=True)
def _library_up_to_date():
    """Rebuild liblocassm.so if any CUDA/C++ source is newer than it (no-op when up to date), so the
    tests never exercise a stale library."""
    from paper_conf_sc_awanhedbdoy21_b200 import build
    build.build()
