import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a CUDA device (B200); parity tests through the C-ABI")
    config.addinivalue_line("markers", "slow: long-running CPU test")
    # Host-side artefacts (generator, oracle) are cheap to (re)build; the CUDA
    # library is built by `make` / __graft_entry__.build().
    subprocess.run(["make", "-s", "-C", ROOT, "tcgen/libtcgen.so", "oracle/libtcoracle.so"],
                   check=True)


def load_edge_file(name):
    """Edge list fixture from tests/golden (see tests/golden/make_golden.py)."""
    import numpy as np
    path = os.path.join(ROOT, "tests", "golden", name)
    rows = [l.split() for l in open(path) if l.strip() and not l.startswith("#")]
    a = np.array([[int(x), int(y)] for x, y in rows], dtype=np.int32)
    return a[:, 0].copy(), a[:, 1].copy()


@pytest.fixture
def golden():
    return load_edge_file
