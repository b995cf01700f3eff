"""pytest configuration: the `gpu` marker and repo-root import path.

`-m "not gpu"` runs the oracle pins, host logic and C-ABI load checks (CPU only);
`-m gpu` runs the CUDA-vs-oracle parity tests through the C ABI on a B200.
"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a CUDA device (B200); parity through the C ABI")
    config.addinivalue_line("markers", "slow: longer CPU oracle runs")
