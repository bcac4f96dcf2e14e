"""Numeric oracle -- TEST INFRASTRUCTURE ONLY.

x = L^{-1} b by Algorithm 1 (section 2.1.1) in fp64, and
x = U^{-1} b by the mirrored backward substitution.  The
recursive-block method reaches exactly this result up to rounding order
(SURVEY.md 8(c)), so the oracle is the plain definition written out.

Pins (tests/test_oracle_numeric.py): closed forms (identity, diagonal, unit
bidiagonal -> prefix sums, geometric bidiagonal, dense all-ones lower ->
first differences), brute-force dense solves (numpy.linalg.solve,
scipy.linalg.solve_triangular) on tiny inputs, the componentwise backward
error bound of substitution, and the pure-Python twin below.
"""
from __future__ import annotations

import ctypes
import time

import numpy as np

from . import build as _build

_lib = None


def lib():
    global _lib
    if _lib is None:
        path = _build.build()
        L = ctypes.CDLL(path)
        L.oracle_trsv.restype = ctypes.c_int
        L.oracle_trsv.argtypes = [ctypes.c_int, ctypes.c_int32, ctypes.c_void_p, ctypes.c_void_p,
                                  ctypes.c_void_p, ctypes.c_int32, ctypes.c_void_p, ctypes.c_int64,
                                  ctypes.c_void_p, ctypes.c_int64, ctypes.c_int32]
        L.oracle_levels.restype = ctypes.c_int32
        L.oracle_levels.argtypes = [ctypes.c_int32, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p]
        _lib = L
    return _lib


def _p(a: np.ndarray):
    return a.ctypes.data_as(ctypes.c_void_p)


def solve(M, b: np.ndarray, threads: int = 1) -> np.ndarray:
    """Solve M x = b for b of numpy shape (nrhs, n) or (n,), in fp64.

    M.uplo == "L": Algorithm 1 (diagonal last in each row).
    M.uplo == "U": backward substitution (diagonal first in each row).
    Returns x with the shape of b (fp64).
    """
    b2 = np.ascontiguousarray(np.atleast_2d(np.asarray(b, dtype=np.float64)))
    nrhs, n = b2.shape
    assert n == M.n
    x = np.zeros_like(b2)
    rp = np.ascontiguousarray(M.row_ptr, dtype=np.int32)
    ci = np.ascontiguousarray(M.col_idx, dtype=np.int32)
    va = np.ascontiguousarray(M.val, dtype=np.float64)
    if n > 0 and nrhs > 0:
        lib().oracle_trsv(1 if M.uplo == "U" else 0, n, _p(rp), _p(ci), _p(va), nrhs,
                          _p(b2), n, _p(x), n, threads)
    return x.reshape(np.shape(b)) if np.ndim(b) == 1 else x


def solve_timed(M, b: np.ndarray, threads: int = 1):
    """(x, seconds, threads_used) for the timed CPU baseline."""
    b2 = np.ascontiguousarray(np.atleast_2d(np.asarray(b, dtype=np.float64)))
    nrhs, n = b2.shape
    x = np.zeros_like(b2)
    rp = np.ascontiguousarray(M.row_ptr, dtype=np.int32)
    ci = np.ascontiguousarray(M.col_idx, dtype=np.int32)
    va = np.ascontiguousarray(M.val, dtype=np.float64)
    t0 = time.perf_counter()
    used = lib().oracle_trsv(1 if M.uplo == "U" else 0, n, _p(rp), _p(ci), _p(va), nrhs,
                             _p(b2), n, _p(x), n, threads)
    dt = time.perf_counter() - t0
    return x, dt, used


def solve_py(M, b) -> np.ndarray:
    """Pure-Python twin of Algorithm 1 / backward substitution (tiny n only)."""
    n = M.n
    rp = [int(v) for v in M.row_ptr]
    ci = [int(v) for v in M.col_idx]
    va = [float(v) for v in M.val]
    bb = [float(v) for v in np.asarray(b, dtype=np.float64).reshape(-1)]
    x = [0.0] * n
    if M.uplo == "L":
        for i in range(n):
            left_sum = 0.0
            for j in range(rp[i], rp[i + 1] - 1):
                left_sum = left_sum + va[j] * x[ci[j]]
            x[i] = (bb[i] - left_sum) / va[rp[i + 1] - 1]
    else:
        for i in range(n - 1, -1, -1):
            left_sum = 0.0
            for j in range(rp[i] + 1, rp[i + 1]):
                left_sum = left_sum + va[j] * x[ci[j]]
            x[i] = (bb[i] - left_sum) / va[rp[i]]
    return np.array(x)


def residual_bound_ok(M, x: np.ndarray, b: np.ndarray, unit_roundoff: float = 2.0 ** -53,
                      slack: float = 2.0):
    """Componentwise backward-error test of a computed solution.

    Substitution in any summation order satisfies (T + dT) x^ = b with
    |dT_ij| <= gamma_{m_i} |T_ij|, m_i = nonzeros of row i (Higham, Accuracy
    and Stability, Thm 8.5 applied per row), hence
        |b - T x^|_i <= gamma_{m_i} (|T| |x^|)_i,  gamma_k = k u / (1 - k u).
    We test with gamma_{m_i+1} and a factor ``slack``.  The residual is
    evaluated in extended precision (np.longdouble) so its own rounding is far
    below the bound.  Returns (ok, worst ratio).
    """
    n = M.n
    x2 = np.atleast_2d(np.asarray(x, dtype=np.float64))
    b2 = np.atleast_2d(np.asarray(b, dtype=np.float64))
    rp = M.row_ptr.astype(np.int64)
    counts = np.diff(rp)
    v = M.val.astype(np.longdouble)
    k = (counts + 1).astype(np.float64)
    gam = k * unit_roundoff / (1.0 - k * unit_roundoff)
    worst = 0.0
    for c in range(x2.shape[0]):
        xc = x2[c].astype(np.longdouble)
        prod = v * xc[M.col_idx]
        # every row holds its diagonal, so no CSR row is empty and reduceat
        # over row_ptr sums exactly the entries of each row
        Tx = np.add.reduceat(prod, rp[:-1]) if n else np.zeros(0, np.longdouble)
        aT = np.add.reduceat(np.abs(prod), rp[:-1]) if n else np.zeros(0, np.longdouble)
        r = np.abs(b2[c].astype(np.longdouble) - Tx).astype(np.float64)
        bound = slack * gam * aT.astype(np.float64)
        with np.errstate(divide="ignore", invalid="ignore"):
            ratio = np.where(bound > 0, r / bound, np.where(r > 0, np.inf, 0.0))
        worst = max(worst, float(ratio.max()) if n else 0.0)
    return worst <= 1.0, worst


def rel_err(x: np.ndarray, x_ref: np.ndarray) -> float:
    """max_c ||x_c - x_ref_c||_inf / ||x_ref_c||_inf."""
    x2 = np.atleast_2d(np.asarray(x, dtype=np.float64))
    r2 = np.atleast_2d(np.asarray(x_ref, dtype=np.float64))
    num = np.abs(x2 - r2).max(axis=1) if x2.shape[1] else np.zeros(x2.shape[0])
    den = np.abs(r2).max(axis=1) if r2.shape[1] else np.ones(r2.shape[0])
    den = np.where(den > 0, den, 1.0)
    return float((num / den).max()) if num.size else 0.0
