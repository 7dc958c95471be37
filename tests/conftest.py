import json
import os
import sys

import numpy as np
import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)

GOLDEN = os.path.join(ROOT, "tests", "golden")


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a CUDA device (B200, sm_100a)")
    config.addinivalue_line("markers", "slow: long-running")


def load_fig2():
    """Fig. 2 matrix (tests/golden/fig2_matrix.txt): returns (nrows, ncols, row, col, val, names)."""
    rows, cols, names = [], [], []
    with open(os.path.join(GOLDEN, "fig2_matrix.txt")) as f:
        for line in f:
            line = line.strip()
            if not line or line.startswith("#"):
                continue
            r, c, nm = line.split()
            rows.append(int(r))
            cols.append(int(c))
            names.append(nm)
    vals = np.array([10.0 * r + c + 1.0 for r, c in zip(rows, cols)])
    return 6, 9, np.array(rows, np.int64), np.array(cols, np.int64), vals, names


def load_fig2_expected():
    with open(os.path.join(GOLDEN, "fig2_crsd.json")) as f:
        return json.load(f)


def fig2_value(name: str) -> float:
    if name == "0":
        return 0.0
    r, c = int(name[1]), int(name[2])
    return 10.0 * r + c + 1.0


@pytest.fixture
def fig2():
    return load_fig2()


@pytest.fixture
def fig2_expected():
    return load_fig2_expected()


def have_gpu() -> bool:
    try:
        import torch

        return torch.cuda.is_available()
    except Exception:
        return False
