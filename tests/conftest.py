"""Shared pytest setup: the `gpu` marker (tests that need a B200; run with
`-m gpu` on the GPU box) and the repo root on sys.path."""
import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a CUDA B200 (run with -m gpu)")
    config.addinivalue_line("markers", "slow: long-running CPU test")


@pytest.fixture(scope="session", autouse=True)
def _oracle_built():
    sys.path.insert(0, os.path.join(ROOT, "tools"))
    from build import build_oracle  # noqa: E402
    build_oracle()
    yield
