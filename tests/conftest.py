import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a B200 (CUDA sm_100a); run with -m gpu")


def rel_errs(got: dict, ref: dict):
    """Per-tensor relative L2 error.  Tensors whose
    reference norm is below 1e-6 of the largest one (e.g. an attention key bias,
    whose gradient is analytically zero by softmax shift invariance) are compared
    against that largest norm instead."""
    import numpy as np
    scale = max(float(np.linalg.norm(np.asarray(v, np.float64))) for v in ref.values())
    out = {}
    for k, r in ref.items():
        r = np.asarray(r, np.float64)
        g = np.asarray(got[k], np.float64).reshape(r.shape)
        den = max(float(np.linalg.norm(r)), 1e-6 * scale)
        out[k] = float(np.linalg.norm(g - r)) / den
    return out
