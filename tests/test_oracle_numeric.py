"""Pins of the numeric oracle (oracle/numeric.py) against facts fixed by the
paper and by mathematics -- not by the oracle itself (CPU only).

Each test is chosen so that a plausible mistake in Algorithm 1's oracle (a
dropped term, the diagonal taken from the wrong end of the row, a wrong sign,
a transposed operand, an off-by-one loop bound) fails at least one of them.
"""
import numpy as np
import pytest
import scipy.linalg

from oracle import numeric as on
from workloads import generators as g


def _dense(M):
    A = np.zeros((M.n, M.n))
    for i in range(M.n):
        for p in range(M.row_ptr[i], M.row_ptr[i + 1]):
            A[i, M.col_idx[p]] = M.val[p]
    return A


def test_identity_returns_b():
    M = g.shape_diagonal(50)
    M.val[:] = 1.0
    b = g.gen_rhs(50, 3, seed=1)
    assert np.array_equal(on.solve(M, b), b)


def test_diagonal_closed_form():
    M = g.shape_diagonal(300)
    b = g.gen_rhs(300, 2, seed=2)
    x = on.solve(M, b)
    # x_i = b_i / d_i: one correctly rounded division, so bit-exact
    assert np.array_equal(x, b / M.val[None, :])


def test_unit_bidiagonal_prefix_sums_exact():
    # sub-diagonal -1, diagonal 1: x_i = sum_{k<=i} b_k; integer b is exact
    n = 2000
    M = g.shape_bidiagonal(n, a=1.0)
    rng = np.random.default_rng(3)
    b = rng.integers(-1000, 1000, size=n).astype(np.float64)
    x = on.solve(M, b)
    assert np.array_equal(x, np.cumsum(b))


def test_geometric_bidiagonal_closed_form():
    # sub-diagonal -a: x_i = sum_k a^(i-k) b_k
    n, a = 200, 0.5
    M = g.shape_bidiagonal(n, a=a)
    b = g.gen_rhs(n, 1, seed=4)[0]
    ref = np.array([sum(a ** (i - k) * b[k] for k in range(i + 1)) for i in range(n)])
    assert np.max(np.abs(on.solve(M, b) - ref)) < 1e-13


def test_dense_all_ones_first_differences():
    # L = all ones lower triangle: L^{-1} is bidiagonal, x_0 = b_0, x_i = b_i - b_{i-1}
    n = 64
    M = g.shape_dense_lower(n)
    M.val[:] = 1.0
    rng = np.random.default_rng(5)
    b = rng.integers(-50, 50, size=n).astype(np.float64)
    x = on.solve(M, b)
    ref = np.concatenate([[b[0]], np.diff(b)])
    assert np.array_equal(x, ref)


@pytest.mark.parametrize("seed", [0, 1, 2])
def test_brute_force_dense_lower(seed):
    M = g.shape_random_small(120, 0.15, seed=seed)
    A = _dense(M)
    b = g.gen_rhs(M.n, 4, seed=seed + 10)
    x = on.solve(M, b)
    ref_np = np.linalg.solve(A, b.T).T
    ref_sp = scipy.linalg.solve_triangular(A, b.T, lower=True).T
    assert on.rel_err(x, ref_np) < 1e-13
    assert on.rel_err(x, ref_sp) < 1e-13


@pytest.mark.parametrize("seed", [0, 1])
def test_brute_force_upper(seed):
    L = g.shape_random_small(90, 0.2, seed=seed)
    U = g.to_upper(L)
    A = _dense(U)
    assert np.allclose(A, np.triu(A))
    b = g.gen_rhs(U.n, 2, seed=seed + 20)
    x = on.solve(U, b)
    ref = scipy.linalg.solve_triangular(A, b.T, lower=False).T
    assert on.rel_err(x, ref) < 1e-13


@pytest.mark.parametrize("seed", [0, 1])
@pytest.mark.parametrize("uplo", ["L", "U"])
def test_brute_force_transposed(seed, uplo):
    """The transposed-solve inputs (R31): transpose() is the dense transpose
    entry for entry, and the oracle's solve of it is a dense solve with A^T."""
    M = g.shape_random_small(80, 0.25, seed=seed + 3)
    if uplo == "U":
        M = g.to_upper(M)
    MT = g.transpose(M)
    assert MT.uplo != M.uplo
    assert np.array_equal(_dense(MT), _dense(M).T)
    T = g.transpose(MT)
    assert np.array_equal(T.row_ptr, M.row_ptr) and np.array_equal(T.col_idx, M.col_idx)
    assert np.array_equal(T.val, M.val)
    b = g.gen_rhs(M.n, 2, seed=seed + 30)
    x = on.solve(MT, b)
    ref = scipy.linalg.solve_triangular(_dense(M), b.T, lower=(uplo == "L"), trans="T").T
    assert on.rel_err(x, ref) < 1e-13


def test_transposed_bidiagonal_suffix_sums():
    """L = unit lower bidiagonal with -1 below the diagonal: L^T x = b is
    x_i = b_i + x_{i+1}, the suffix sums (exact in integers)."""
    n = 400
    L = g.shape_bidiagonal(n, a=1.0)
    rng = np.random.default_rng(9)
    b = rng.integers(-9, 9, size=n).astype(np.float64)
    assert np.array_equal(on.solve(g.transpose(L), b), np.cumsum(b[::-1])[::-1])


def test_upper_bidiagonal_suffix_sums():
    n = 500
    U = g.to_upper(g.shape_bidiagonal(n, a=1.0))
    rng = np.random.default_rng(6)
    b = rng.integers(-9, 9, size=n).astype(np.float64)
    assert np.array_equal(on.solve(U, b), np.cumsum(b[::-1])[::-1])


def test_python_twin_agrees_bitwise():
    M = g.c1_random(n=300)
    b = g.gen_rhs(M.n, 1, seed=7)[0]
    assert np.array_equal(on.solve(M, b), on.solve_py(M, b))
    U = g.to_upper(M)
    assert np.array_equal(on.solve(U, b), on.solve_py(U, b))


def test_multi_rhs_columns_independent_and_threaded():
    M = g.c5_random_multirhs(n=3000)
    b = g.gen_rhs(M.n, 9, seed=8)
    x1 = on.solve(M, b, threads=1)
    x4 = on.solve(M, b, threads=4)
    assert np.array_equal(x1, x4)
    for c in (0, 5, 8):
        assert np.array_equal(x1[c], on.solve(M, b[c]))


@pytest.mark.parametrize("name", ["C1", "C2", "C3", "C4", "C5"])
def test_backward_error_invariant_small_configs(name):
    M, b = g.gen_config(name, small=True, nrhs=2)
    x = on.solve(M, b)
    ok, worst = on.residual_bound_ok(M, x, b)
    assert ok, worst


def test_backward_error_detects_wrong_solution():
    M, b = g.gen_config("C1", nrhs=1)
    x = on.solve(M, b)
    x[0, 500] *= 1 + 1e-9
    ok, _ = on.residual_bound_ok(M, x, b)
    assert not ok


def test_normwise_residual():
    M, b = g.gen_config("C2", small=True)
    x = on.solve(M, b)
    A_x = np.zeros(M.n)
    rows = np.repeat(np.arange(M.n), np.diff(M.row_ptr))
    np.add.at(A_x, rows, M.val * x[0][M.col_idx])
    assert np.abs(b[0] - A_x).max() / np.abs(b[0]).max() < M.n * 2.0 ** -53


def test_rel_err_definition():
    ref = np.array([[1.0, -2.0, 4.0]])
    x = np.array([[1.0, -2.0, 4.0 + 4e-10]])
    assert abs(on.rel_err(x, ref) - 1e-10) < 1e-15


def test_rhs_column_shards_match_full_draw():
    """bench.py / dist ranks draw only their RHS columns (PCG64 jump-ahead);
    they must be byte-identical to the corresponding columns of gen_rhs."""
    from workloads import generators as g
    full = g.gen_rhs(997, 9, seed=123)
    for c0, c1 in [(0, 9), (0, 1), (3, 7), (8, 9)]:
        assert np.array_equal(g.gen_rhs_cols(997, c0, c1, seed=123), full[c0:c1])
