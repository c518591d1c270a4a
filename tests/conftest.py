"""Shared pytest setup.

Markers: ``gpu`` -- needs a B200 (sm_100a) and the built CUDA library; everything else runs on CPU.
"""
import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: requires a CUDA B200 GPU and the built libseastar.so")
    config.addinivalue_line("markers", "slow: large sizes (still CPU-only unless also marked gpu)")


def rel_err(got, ref):
    """max|got - ref| / max|ref|  (max-abs normalised, the north_star tolerance metric)."""
    import numpy as np
    got = np.asarray(got, np.float64)
    ref = np.asarray(ref, np.float64)
    assert got.shape == ref.shape, (got.shape, ref.shape)
    if ref.size == 0:
        return 0.0
    den = np.abs(ref).max()
    num = np.abs(got - ref).max()
    if den == 0.0:
        return float(num)
    return float(num / den)
