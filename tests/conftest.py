"""pytest configuration: the `gpu` marker and repo-root import path.

-m "not gpu" runs here (no GPU): oracle pins, host logic, C-ABI loading,
gloo world_size-2 tests. -m gpu runs on a B200 through gpurun.
"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a CUDA B200 (runs under gpurun)")
    config.addinivalue_line("markers", "slow: longer CPU test")
