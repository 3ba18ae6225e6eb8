import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a B200 (sm_100a) and the CUDA library")
    config.addinivalue_line("markers", "slow: long-running CPU test")


@pytest.fixture(scope="session")
def xs_small():
    import gen
    return gen.XSTables(**gen.XS_SMALL)


@pytest.fixture(scope="session")
def rs_tables():
    import gen
    return gen.RSTables()


@pytest.fixture(scope="session")
def rs_tables_small():
    """A reduced RSBench shape (fewer nuclides/poles) for fast parity runs."""
    import gen
    return gen.RSTables(n_nuclides=355, avg_poles=100, avg_windows=10)


@pytest.fixture(scope="session")
def rt():
    """The CUDA library, initialized on cuda:0 (GPU tests only; no fallback)."""
    import torch
    from paper_conf_ipps_doerfertphtdcg22_b200 import build, omprt
    if not torch.cuda.is_available():
        pytest.fail("GPU test run without a GPU")
    build.build()
    torch.cuda.set_device(0)
    omprt.omprt_init(0)
    return omprt
