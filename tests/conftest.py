import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a CUDA device (B200) and the built libdgr.so")
    config.addinivalue_line("markers", "slow: longer CPU test")

# the oracle evaluates octant-to-patch + RHS on forked workers (bitwise the same)
os.environ.setdefault("DGR_ORACLE_WORKERS", str(min(16, len(os.sched_getaffinity(0)))))
