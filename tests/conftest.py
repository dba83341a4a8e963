"""pytest configuration: the `gpu` marker and the native build.

`-m "not gpu"` tests run here on CPU (oracle pins, host logic, ABI exports,
gloo multi-process); `-m gpu` tests need a B200 and call the CUDA path through
the C-ABI (libsand.so).
"""
import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a CUDA device (B200, sm_100a)")


@pytest.fixture(scope="session", autouse=True)
def _native_build():
    import native_build
    native_build.build_synth()
    native_build.build_oracle()
    if os.path.isdir(native_build.CSRC):
        native_build.build_product()
    yield
