"""pytest configuration: the `gpu` marker and an in-tree build of the native libraries.

`-m "not gpu"` runs here (no GPU): the oracle against its pins, the generator,
host logic and the C-ABI symbol checks.  `-m gpu` runs on a B200 via gpurun:
the CUDA path (through the C-ABI) against the oracle.
"""
import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a CUDA device (B200); run under gpurun")
    config.addinivalue_line("markers", "slow: long-running CPU test")


@pytest.fixture(scope="session", autouse=True)
def _built():
    sys.path.insert(0, os.path.join(ROOT, "scripts"))
    import build  # noqa: E402

    build.build_oracle()
    build.build_oracle_par()
    build.build_inlgen()
    import glob
    if glob.glob(os.path.join(ROOT, "paper_conf_icpp_liwb15_b200", "csrc", "*.cu")):
        build.build_inl()
    yield


def cuda_ok() -> bool:
    try:
        import torch
        return torch.cuda.is_available()
    except Exception:
        return False


@pytest.fixture
def cuda():
    if not cuda_ok():
        pytest.fail("gpu test selected but no CUDA device is visible")
    import torch
    return torch.device("cuda", 0)
