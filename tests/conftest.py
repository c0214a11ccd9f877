"""Test configuration.

Markers: ``gpu`` -- needs a B200 and the CUDA library (run under gpurun).
Everything else runs on CPU (oracle pins, generators, host logic, ABI load).
"""
import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a CUDA device (B200) and libnest.so")
    config.addinivalue_line("markers", "slow: long-running CPU test")
    # host libraries (generators + oracle) are plain gcc builds; make is a no-op when fresh
    subprocess.run(["make", "-s", "-C", ROOT, "host"], check=True)


def pytest_collection_modifyitems(config, items):
    for item in items:
        if "gpu" in item.keywords:
            item.add_marker(pytest.mark.timeout(900))
