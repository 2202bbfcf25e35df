import os
import sys
from pathlib import Path

import pytest

ROOT = Path(__file__).resolve().parents[1]
sys.path.insert(0, str(ROOT))
sys.path.insert(0, str(Path(__file__).resolve().parent))


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a CUDA device (B200, sm_100a)")
    config.addinivalue_line("markers", "slow: full-size configurations")


def pytest_collection_modifyitems(config, items):
    # a gpu test on a box without a GPU must fail loudly, never silently skip
    # into a CPU path; but the CPU suite is selected with -m "not gpu".
    pass
