import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a B200 (sm_100a) and the built CUDA library")
    config.addinivalue_line("markers", "slow: long-running CPU test")


def load_golden(name):
    """Parse a tests/golden/*.txt matrix fixture into a dict of numpy arrays."""
    import numpy as np
    mats, cur, rows = {}, None, []
    with open(os.path.join(ROOT, "tests", "golden", name)) as f:
        for line in f:
            line = line.strip()
            if not line or line.startswith("#"):
                continue
            parts = line.split()
            if parts[0].isalpha():
                cur, r, c = parts[0], int(parts[1]), int(parts[2])
                mats[cur] = np.zeros((r, c), dtype=np.float64)
                rows = [0]
                continue
            mats[cur][rows[0]] = [float(x) for x in parts]
            rows[0] += 1
    return mats
