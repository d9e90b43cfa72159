import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a CUDA device (B200); parity tests through the C ABI")
    config.addinivalue_line("markers", "slow: full-size (Europe/USA-scale) cases")
    # Build the host libraries if a fresh checkout has none (cheap; gcc only).
    need = [os.path.join(ROOT, "phastgen", "libphastgen.so"), os.path.join(ROOT, "oracle", "liboracle.so")]
    if not all(os.path.exists(p) for p in need):
        import __graft_entry__
        __graft_entry__.build_c()


@pytest.fixture(scope="session")
def root():
    return ROOT
