import os
import sys

import numpy as np
import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a CUDA B200 (sm_100a) and the built libtqr.so")
    config.addinivalue_line("markers", "slow: long-running (large sizes)")


def sign_normalise_R(R):
    """D R with D = diag(sgn R_ii), sgn(0) = +1  (reading Q17)."""
    R = np.array(R, dtype=np.float64)
    d = np.where(np.diag(R) < 0, -1.0, 1.0)
    return R * d[:, None]


def colnorm_rel_err(R_test, R_ref):
    """max_ij |R~_ij - R^_ij| / ||R^(:, j)||_2 after sign normalisation (reading Q16)."""
    a = sign_normalise_R(R_test)
    b = sign_normalise_R(R_ref)
    cn = np.linalg.norm(b, axis=0)
    cn[cn == 0] = 1.0
    return float(np.max(np.abs(a - b) / cn[None, :])) if a.size else 0.0


@pytest.fixture
def golden_dir():
    return os.path.join(ROOT, "tests", "golden")
