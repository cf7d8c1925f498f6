"""oracle -- TEST INFRASTRUCTURE ONLY (never imported by the product package).

Plain CPU fp64 reference of what the tiled-QR hot path computes, written from
Kim & Park, "Tiled QR Decomposition and Its Optimization on CPU and GPU Computing
System", ICPP'13:

* ``qr``            -- Algorithm 1, Householder QR (P:L228-240 + P:L203-211), in
                       ``householder.c`` (plain C, no blocking).
* ``apply_q``       -- Q^T B / Q B from the same reflectors (Alg. 1 lines 13-14).
* ``solve_ls``      -- Eqs. (2)-(3): R x = Q^T b.
* ``guide.generate_array`` / ``guide.distribute`` -- Algorithm 4 + Eq. (12).

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py`` (cpu_baseline leg and
``--impl reference``) may import this package.  It shares no code with
``paper_conf_icpp_kimp13_b200``; the shared seeded input generator lives in
``synthetic/`` and holds none of the method's arithmetic.

Pins (tests/test_oracle.py): closed-form 2x2, the textbook 3x3 (exact Q and R),
50-digit mpmath Gram-Schmidt on tiny inputs, R^T R = A^T A, |det A| = prod |R_ii|,
orthogonal / triangular / diagonal special cases, LAPACK (numpy.linalg.qr) agreement,
and the paper's worked guide-array example.  Nothing here is
"parity unpinned" except where DESIGN.md says so.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
import threading

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "householder.c")
_LIB = os.path.join(_HERE, "liboracle.so")
_lock = threading.Lock()
_lib = None


def build(force: bool = False) -> str:
    """Compile householder.c -> liboracle.so with gcc (plain -O2, no fast-math, no FMA contraction)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + ".%d.tmp" % os.getpid()
        subprocess.check_call(["gcc", "-O2", "-fopenmp", "-ffp-contract=off", "-fno-fast-math",
                               "-shared", "-fPIC", "-o", tmp, _SRC, "-lm"])
        os.replace(tmp, _LIB)
    return _LIB


def _load():
    global _lib
    with _lock:
        if _lib is None:
            build()
            lib = ctypes.CDLL(_LIB)
            i64, i32, dp = ctypes.c_int64, ctypes.c_int, ctypes.POINTER(ctypes.c_double)
            lib.oracle_qr.argtypes = [i64, i64, dp, i64, dp, i64, i32]
            lib.oracle_qr.restype = None
            lib.oracle_apply_q.argtypes = [i64, i64, dp, i64, dp, i64, i64, ctypes.c_char, i32]
            lib.oracle_apply_q.restype = None
            lib.oracle_back_substitute.argtypes = [i64, dp, i64, dp, i64, i64]
            lib.oracle_back_substitute.restype = i64
            lib.oracle_num_threads.argtypes = []
            lib.oracle_num_threads.restype = i32
            _lib = lib
    return _lib


def _ptr(a: np.ndarray):
    return a.ctypes.data_as(ctypes.POINTER(ctypes.c_double))


def _colmajor(a) -> np.ndarray:
    return np.asfortranarray(np.asarray(a, dtype=np.float64)).copy(order="F")


def num_threads() -> int:
    return int(_load().oracle_num_threads())


class Factorization:
    """Result of Algorithm 1: R (n x n upper triangular) and the unit reflectors V (m x n)."""

    def __init__(self, R: np.ndarray, V: np.ndarray, m: int, n: int):
        self.R, self.V, self.m, self.n = R, V, m, n

    def apply_q(self, B, trans: str = "T", nthreads: int = 0) -> np.ndarray:
        return apply_q(self.V, B, trans, nthreads)

    def thin_q(self, nthreads: int = 0) -> np.ndarray:
        """Q[:, :n] = Q [I_n; 0]  (Alg. 1 line 13 applied to the first n unit vectors)."""
        E = np.zeros((self.m, self.n), order="F")
        E[: self.n, : self.n] = np.eye(self.n)
        return apply_q(self.V, E, "N", nthreads)


def qr(A, nthreads: int = 0) -> Factorization:
    """Algorithm 1 on A (m x n, m >= n).  Returns R = triu(Q^T A)[:n, :n] and the reflectors."""
    A = _colmajor(A)
    if A.ndim != 2:
        raise ValueError("A must be 2-D")
    m, n = A.shape
    if m < n:
        raise ValueError("oracle.qr needs m >= n")
    V = np.zeros((m, n), order="F")
    if n:
        _load().oracle_qr(m, n, _ptr(A), max(m, 1), _ptr(V), max(m, 1), int(nthreads))
    R = np.triu(A[:n, :n])
    return Factorization(R, V, m, n)


def qr_columns(A, ncols: int, nthreads: int = 0) -> np.ndarray:
    """Run only the first ``ncols`` iterations of Algorithm 1 (bounded CPU-baseline samples).

    This is Algorithm 1 on the full matrix stopped after column ``ncols``; it is used by
    bench.py to time a bounded, representative sample of the oracle's work.
    """
    A = _colmajor(A)
    m, n = A.shape
    V = np.zeros((m, ncols), order="F")
    _load().oracle_qr(m, ncols, _ptr(A), max(m, 1), _ptr(V), max(m, 1), int(nthreads))
    # columns >= ncols received Q_0..Q_{ncols-1} only through the apply below
    rest = np.asfortranarray(A[:, ncols:])
    _load().oracle_apply_q(m, ncols, _ptr(V), max(m, 1), _ptr(rest), max(m, 1), n - ncols, b"T", int(nthreads))
    A[:, ncols:] = rest
    return A


def apply_q(V, B, trans: str = "T", nthreads: int = 0) -> np.ndarray:
    """B <- Q^T B (trans 'T') or Q B (trans 'N') using Algorithm 1's reflectors."""
    V = _colmajor(V)
    B = _colmajor(B)
    squeeze = B.ndim == 1
    if squeeze:
        B = B.reshape(-1, 1, order="F")
    m, n = V.shape
    if B.shape[0] != m:
        raise ValueError("row mismatch")
    nrhs = B.shape[1]
    if nrhs and n:
        _load().oracle_apply_q(m, n, _ptr(V), max(m, 1), _ptr(B), max(m, 1), nrhs,
                               trans.encode()[:1], int(nthreads))
    return B[:, 0] if squeeze else B


def solve_ls(A, B, nthreads: int = 0) -> np.ndarray:
    """Least squares via Eqs. (2)-(3): x = R^{-1} (Q^T b)[:n]."""
    f = qr(A, nthreads)
    C = apply_q(f.V, B, "T", nthreads)
    squeeze = C.ndim == 1
    if squeeze:
        C = C.reshape(-1, 1, order="F")
    X = np.asfortranarray(C[: f.n, :]).copy(order="F")
    R = np.asfortranarray(f.R)
    bad = _load().oracle_back_substitute(f.n, _ptr(R), max(f.n, 1), _ptr(X), max(f.n, 1), X.shape[1])
    if bad:
        raise ZeroDivisionError("R[%d,%d] == 0" % (bad - 1, bad - 1))
    return X[:, 0] if squeeze else X


from . import guide  # noqa: E402  (Algorithm 4 / Eq. 12, pure Python)

__all__ = ["build", "qr", "qr_columns", "apply_q", "solve_ls", "Factorization", "guide", "num_threads"]
