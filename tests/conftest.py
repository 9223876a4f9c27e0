"""pytest configuration: the `gpu` marker and import paths.

Tests marked ``@pytest.mark.gpu`` need a B200 (sm_100a); everything else runs
on CPU (the oracle pins, the layout compiler through the C-ABI's host-only
calls, the planner, the symbol table, the gloo multi-process tests).
"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a CUDA B200 (sm_100a) device")
