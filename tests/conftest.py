import os
import sys

import numpy as np
import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)

GOLDEN = os.path.join(ROOT, "tests", "golden")


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a B200 (runs through libbar.so's C-ABI)")
    config.addinivalue_line("markers", "slow: larger CPU cases")
    from tools.build import build_oracle, build_workloads

    build_workloads()
    build_oracle()


def load_golden(name):
    """Whitespace table under tests/golden/ (comment lines start with '#')."""
    rows = []
    with open(os.path.join(GOLDEN, name)) as f:
        for line in f:
            line = line.strip()
            if not line or line.startswith("#"):
                continue
            rows.append(line.split())
    return rows


@pytest.fixture(scope="session")
def golden():
    return load_golden


@pytest.fixture(scope="session")
def bar():
    """The CUDA path through the C-ABI; GPU tests only."""
    import torch

    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    from paper_conf_ipps_anzttdh12_b200 import bar as _bar

    return _bar


@pytest.fixture()
def rng():
    return np.random.default_rng(0)
