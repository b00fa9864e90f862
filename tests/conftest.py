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
    reference norm is below 1e-4 of the largest one (e.g. an attention key bias,
    whose gradient is analytically zero by softmax shift invariance, so fp32
    cancellation noise is all that is left) are compared against 1e-4 x the
    largest norm instead."""
    import numpy as np
    scale = max(float(np.linalg.norm(np.asarray(v, np.float64))) for v in ref.values())
    out = {}
    for k, r in ref.items():
        r = np.asarray(r, np.float64)
        g = np.asarray(got[k], np.float64).reshape(r.shape)
        den = max(float(np.linalg.norm(r)), 1e-4 * scale)
        out[k] = float(np.linalg.norm(g - r)) / den
    return out


def global_rel_err(got: dict, ref: dict):
    """Relative L2 error of the whole gradient vector (all parameters
    concatenated): DESIGN.md reading D-TOL for bf16 runs."""
    import numpy as np
    num = sum(float(np.sum((np.asarray(got[k], np.float64).reshape(np.shape(r)) - np.asarray(r, np.float64)) ** 2))
              for k, r in ref.items())
    den = sum(float(np.sum(np.asarray(r, np.float64) ** 2)) for r in ref.values())
    return (num / den) ** 0.5


BF16_TOL = 2e-2  # north_star: bf16 gradients within 2e-2 of the fp64 oracle (per tensor, R17)


def assert_bf16_parity(got: dict, ref: dict, tol: float = BF16_TOL):
    """Per-tensor relative L2 <= tol against the plain fp64 oracle (`net.train_step`,
    storage=None), with rel_errs' floor for analytically-zero tensors."""
    errs = rel_errs(got, ref)
    worst = sorted(errs.items(), key=lambda kv: -kv[1])[:5]
    assert worst[0][1] <= tol, worst
    return errs
