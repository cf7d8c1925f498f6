"""synthetic -- seeded input generators shared by tests, bench.py and smoke().

Holds none of the method's arithmetic: it only draws matrices.  The paper's workload is
"random floating point numbers" in square matrices (Table III P:L1329-1521,
Fig. 8); BASELINE.json fixes iid N(0,1) (reading Q10).

``gaussian(m, n, seed)`` is counter based: A(i, j) = Box-Muller(SplitMix64(seed, i + j*m)),
so any sub-block can be regenerated independently (used for sampled full-size checks) and
the value does not depend on numpy's RNG version.  Column-major (Fortran) order.
"""
from __future__ import annotations

import numpy as np

_M64 = np.uint64(0xFFFFFFFFFFFFFFFF)


def _splitmix64(x: np.ndarray) -> np.ndarray:
    with np.errstate(over="ignore"):
        z = x + np.uint64(0x9E3779B97F4A7C15)
        z = (z ^ (z >> np.uint64(30))) * np.uint64(0xBF58476D1CE4E5B9)
        z = (z ^ (z >> np.uint64(27))) * np.uint64(0x94D049BB133111EB)
        return z ^ (z >> np.uint64(31))


def _uniform01(bits: np.ndarray) -> np.ndarray:
    # 53 random bits -> (0, 1]
    return ((bits >> np.uint64(11)).astype(np.float64) + 1.0) * (1.0 / 9007199254740992.0)


def gaussian_counter(counter: np.ndarray, seed: int) -> np.ndarray:
    """N(0,1) value for each 64-bit counter (Box-Muller on two SplitMix64 draws)."""
    c = counter.astype(np.uint64)
    with np.errstate(over="ignore"):
        key = _splitmix64(np.uint64(seed) * np.uint64(0xD1B54A32D192ED03) + np.uint64(1))
        b1 = _splitmix64(key ^ (c * np.uint64(2)))
        b2 = _splitmix64(key ^ (c * np.uint64(2) + np.uint64(1)))
    u1, u2 = _uniform01(b1), _uniform01(b2)
    return np.sqrt(-2.0 * np.log(u1)) * np.cos(2.0 * np.pi * u2)


def gaussian(m: int, n: int, seed: int) -> np.ndarray:
    """m x n column-major iid N(0,1) fp64 matrix, A(i,j) = f(seed, i + j*m)."""
    idx = np.arange(m * n, dtype=np.uint64)
    return gaussian_counter(idx, seed).reshape((m, n), order="F")


def gaussian_entries(m: int, rows: np.ndarray, cols: np.ndarray, seed: int) -> np.ndarray:
    """Entries A(rows[k], cols[k]) of gaussian(m, n, seed) without materialising A."""
    idx = rows.astype(np.uint64) + cols.astype(np.uint64) * np.uint64(m)
    return gaussian_counter(idx, seed)


def ill_conditioned(m: int, n: int, seed: int, cond: float = 1e10) -> np.ndarray:
    """U diag(sigma) V^T with sigma geometric from 1 to 1/cond (correctness-only input)."""
    rng = np.random.Generator(np.random.PCG64(seed))
    U, _ = np.linalg.qr(rng.standard_normal((m, n)))
    W, _ = np.linalg.qr(rng.standard_normal((n, n)))
    sig = np.geomspace(1.0, 1.0 / cond, n)
    return np.asfortranarray((U * sig) @ W.T)


def integer_matrix(m: int, n: int, seed: int, lo: int = -9, hi: int = 9) -> np.ndarray:
    rng = np.random.Generator(np.random.PCG64(seed))
    return np.asfortranarray(rng.integers(lo, hi + 1, size=(m, n)).astype(np.float64))


# BASELINE.json configs: name -> (m, n, nb, ib, seed)
CONFIGS = {
    "C1": dict(m=256, n=256, nb=64, ib=16, seed=101),
    "C2": dict(m=4096, n=4096, nb=256, ib=32, seed=102),
    "C3": dict(m=16384, n=16384, nb=512, ib=32, seed=103),
    "C4": dict(m=1048576, n=512, nb=512, ib=32, seed=104),
    "C5": dict(m=32768, n=32768, nb=512, ib=32, seed=105),
}
