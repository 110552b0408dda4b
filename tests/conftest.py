import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a B200 (run through gpurun)")
    config.addinivalue_line("markers", "slow: long-running CPU oracle check")


import pytest  # noqa: E402


@pytest.fixture(scope="session")
def mxlib():
    """Initialise libmx.so once per test session on GPU 0 (GPU tests only)."""
    from paper_conf_sc_dhakalrwercfm23_b200 import mx
    mx.mx_init([0])
    yield mx
    mx.mx_shutdown()


@pytest.fixture()
def parts(mxlib):
    """Create partitions inside a test; destroyed (after their tasks are waited) at the end."""
    created = []

    def make(sm, hbm=1 << 30, gpu=0):
        p = mxlib.part_create(gpu, sm, hbm)
        created.append(p)
        return p

    yield make
    for p in created:
        try:
            mxlib.part_destroy(p)
        except Exception:
            pass
