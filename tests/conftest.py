import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a real B200 (CUDA path through the C ABI)")
    config.addinivalue_line("markers", "slow: long-running")


def cuda_available():
    try:
        import torch
        return torch.cuda.is_available()
    except Exception:
        return False


@pytest.fixture(scope="session")
def golden_dir():
    return os.path.join(ROOT, "tests", "golden")


def import_tiles():
    """The native binding. On a GPU box a missing or broken libtiles.so is an
    ERROR (no silent skip: the CUDA path must be the one that runs); on a
    CPU-only host the GPU-marked modules skip."""
    if cuda_available():
        from paper_conf_icpp_bastemuzas17_b200 import tiles
        return tiles
    return pytest.importorskip("paper_conf_icpp_bastemuzas17_b200.tiles")
