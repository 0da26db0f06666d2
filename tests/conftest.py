import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)

GOLDEN = os.path.join(ROOT, "tests", "golden")


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a CUDA B200 (run via gpurun)")
    config.addinivalue_line("markers", "slow: long-running (large sizes)")


def load_matrix(name):
    rows = []
    with open(os.path.join(GOLDEN, name)) as f:
        for line in f:
            line = line.strip()
            if not line or line.startswith("#"):
                continue
            rows.append([int(x) for x in line.split()])
    return rows


def load_keyed(name):
    out = {}
    with open(os.path.join(GOLDEN, name)) as f:
        for line in f:
            line = line.strip()
            if not line or line.startswith("#"):
                continue
            k, *vals = line.split()
            out[k] = [int(x) for x in vals]
    return out


@pytest.fixture(scope="session")
def fig3():
    import numpy as np
    a = np.array(load_matrix("fig3_input.txt"), dtype=np.int32)
    cp = np.array(load_matrix("fig3_colprefix.txt"), dtype=np.int32)
    b = np.array(load_matrix("fig3_sat.txt"), dtype=np.int32)
    return a, cp, b
