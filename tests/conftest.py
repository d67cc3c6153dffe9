"""Shared pytest setup: repo root on sys.path, the `gpu` marker, oracle build."""
import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)

# The native libraries are git-ignored build products (__graft_entry__.build() makes them);
# a checkout tested before building gets the runtime and its test library built here
# (up-to-date builds are skipped).  The nvcc AOT library is left to build().
_PKG = os.path.join(ROOT, "paper_conf_cgo_georgakoudispb25_b200")
if not all(os.path.exists(os.path.join(_PKG, f))
           for f in ("libproteus.so", "libproteus_testing.so")):
    from paper_conf_cgo_georgakoudispb25_b200 import _build
    _build.build_runtime()


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a CUDA device (B200, sm_100a)")
    config.addinivalue_line("markers", "slow: long-running CPU test")


@pytest.fixture(scope="session")
def orc():
    import oracle
    oracle.build()
    return oracle
