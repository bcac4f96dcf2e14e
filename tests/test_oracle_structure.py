"""Pins of the structural oracle (oracle/structure.py) against the paper's
text, closed forms and brute force (CPU only)."""
import os

import numpy as np
import pytest
import scipy.sparse as sp

from oracle import numeric as on
from oracle import structure as st
from workloads import generators as g

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def _local_csr(M):
    return M.row_ptr.astype(np.int64), M.col_idx


def _scipy(M):
    return sp.csr_matrix((M.val, M.col_idx, M.row_ptr), shape=(M.n, M.n))


# --------------------------------------------------------------------- levels
def test_paper_fig1_levels_golden():
    want = {}
    for line in open(os.path.join(GOLDEN, "paper_fig1_levels.txt")):
        line = line.strip()
        if not line or line.startswith("#"):
            continue
        lv, comps = line.split(":")
        for c in comps.split():
            want[int(c)] = int(lv)
    M = g.shape_paper_fig1()
    assert M.nnz == 15  # PAPER.md:L73 "L of 15 nonzeros"
    for fn in (st.levels_sweep, st.levels_peel):
        lev, nl = fn(M.n, *_local_csr(M))
        assert nl == 4
        assert [int(v) for v in lev] == [want[i] for i in range(8)]


@pytest.mark.parametrize("seed", range(6))
def test_sweep_equals_alg2_peel(seed):
    M = g.shape_random_small(70 + 13 * seed, [0.02, 0.05, 0.1, 0.3, 0.6, 0.9][seed], seed)
    a, na = st.levels_sweep(M.n, *_local_csr(M))
    b, nb = st.levels_peel(M.n, M.row_ptr, M.col_idx)
    assert na == nb and np.array_equal(a, b)


def test_levels_special_cases():
    assert st.levels_sweep(100, *_local_csr(g.shape_diagonal(100)))[1] == 1
    lev, nl = st.levels_sweep(333, *_local_csr(g.shape_bidiagonal(333)))
    assert nl == 333 and np.array_equal(lev, np.arange(333))
    lev, nl = st.levels_sweep(40, *_local_csr(g.shape_dense_lower(40)))
    assert nl == 40
    lev, nl = st.levels_sweep(50, *_local_csr(g.shape_arrow(50)))
    assert nl == 3 and lev[0] == 0 and lev[-1] == 2 and np.all(lev[1:-1] == 1)
    assert st.levels_sweep(0, np.zeros(1, np.int64), np.zeros(0, np.int32))[1] == 0


def test_c2_levels_closed_form():
    nx, ny = 157, 131
    M = g.c2_laplacian_ic0(nx, ny)
    lev, nl = st.levels_sweep(M.n, *_local_csr(M))
    i = np.arange(M.n)
    assert nl == nx + ny - 1
    assert np.array_equal(lev, (i % nx) + (i // nx))
    mn, avg, mx = st.level_stats(lev, nl)
    assert (mn, avg, mx) == (1, M.n // nl, min(nx, ny))


def test_c3_levels_by_construction():
    M = g.c3_powerlaw_layers(n=40_000, P=61)
    lev, nl = st.levels_sweep(M.n, *_local_csr(M))
    assert nl == 61
    want = np.repeat(np.arange(61), M.meta["level_widths"])
    assert np.array_equal(lev, want)


# PAPER.md:L329-L334 (Table 4): n, #level-sets, parallelism min / ave. / max as printed
TABLE4 = [
    ("nlpkkt200", 16240000, 2, 8000000, 8120000, 8240000),
    ("mawi_201512020030", 68863315, 19, 11, 3624385, 34544376),
    ("kkt_power", 2063494, 17, 1090, 121382, 626597),
    ("FullChip", 2987012, 324, 1, 9219, 468405),
    ("vas_stokes_4M", 4382246, 2815, 1, 1556, 37519),
    ("tmt_sym", 726713, 726235, 1, 1, 135),
]


def _levels_with_sizes(n, nl, mn, mx):
    """A level vector of n rows in nl levels whose smallest level has mn rows
    and whose largest has mx rows (the rest filled greedily within [mn, mx])."""
    sizes = np.full(nl, mn, dtype=np.int64)
    sizes[-1] = mx
    rest = n - sizes.sum()
    assert rest >= 0
    i = 1
    while rest > 0:
        add = min(rest, mx - sizes[i])
        sizes[i] += add
        rest -= add
        i += 1
    assert sizes.sum() == n and sizes.min() == mn and sizes.max() == mx
    return np.repeat(np.arange(nl, dtype=np.int32), sizes)


@pytest.mark.parametrize("row", TABLE4, ids=[r[0] for r in TABLE4])
def test_table4_level_stats_reproduce_printed_parallelism(row):
    """level_stats against every Table 4 row: a level
    vector with the printed n, #level-sets and min / max widths must give the
    printed 'ave.' -- floor(n / #levels): FullChip (9219.2) and vas_stokes_4M
    (1556.7) separate floor from rounding."""
    _name, n, nl, mn, ave, mx = row
    lev = _levels_with_sizes(n, nl, mn, mx)
    assert st.level_stats(lev, nl) == (mn, ave, mx)


def test_table4_average_parallelism_convention():
    lev = np.array([0, 0, 0, 1, 1, 2, 3], dtype=np.int32)
    assert st.level_stats(lev, 4) == (1, 1, 3)


# ------------------------------------------------------------- depth rule
def test_depth_rule_paper_example():
    T = st.paper_threshold(4608)
    assert T == 92160
    assert st.depth_rule(92160, T) == 0
    assert st.depth_rule(184319, T) == 0
    assert st.depth_rule(184320, T) == 1
    assert st.depth_rule(1_000_000, T) == 3
    B200 = st.paper_threshold(148 * 128)
    assert B200 == 378880
    assert st.depth_rule(1_000_000, B200) == 1  # C2
    assert st.depth_rule(4_000_000, B200) == 3  # C3
    assert st.depth_rule(500_000, B200) == 0  # C4
    assert st.depth_rule(2_000_000, B200) == 2  # C5


@pytest.mark.parametrize("d", [0, 1, 2, 5])
def test_recursion_counts(d):
    # depth 2 -> four triangles and three squares
    segs = st.partition(1000, d, "REC")
    assert sum(s.kind == "TRI" for s in segs) == 2 ** d
    assert sum(s.kind == "SQ" for s in segs) == 2 ** d - 1
    kinds = [s.kind for s in segs]
    assert kinds == (["TRI", "SQ"] * (2 ** d))[:-1]  # alternate in execution order (L229)


def test_tables_1_2_exact_and_printed():
    rows = {}
    for line in open(os.path.join(GOLDEN, "tables_1_2.txt")):
        if line.startswith("#") or not line.strip():
            continue
        t, m, _f, *vals = line.split()
        rows[(t, m)] = [float(v) for v in vals]
    n = 2 ** 20
    for xi, x in enumerate([2, 4, 8, 16]):
        for m in ("COL", "ROW", "REC"):
            b_upd, x_ld = st.dense_counts(n, x, m)
            exact_b = {"COL": (2 ** (x - 1) + 0.5) * n, "ROW": (2 - 2.0 ** -x) * n,
                       "REC": (0.5 * x + 1) * n}[m]
            exact_x = {"COL": (1 - 2.0 ** -x) * n, "ROW": (2 ** (x - 1) - 0.5) * n,
                       "REC": 0.5 * x * n}[m]
            assert b_upd == exact_b and x_ld == exact_x, (m, x)
            assert abs(b_upd / n - rows[("T1", m)][xi]) <= 0.01 + 1e-12
            assert abs(x_ld / n - rows[("T2", m)][xi]) <= 0.01 + 1e-12


# ---------------------------------------------------------------- Alg 7
def test_alg7_triangle_boundaries():
    S = st
    assert S.select_tri(1, 1) == S.TRI_COMPLETELY_PARALLEL
    assert S.select_tri(1, 40) == S.TRI_COMPLETELY_PARALLEL
    assert S.select_tri(20001, 1) == S.TRI_NEAR_SERIAL
    # 20000 levels at nnz/row 1: not <= 100 levels (first level-set branch), not
    # <= 20 levels (second), not > 20000 (near-serial) -> Sync-free
    assert S.select_tri(20000, 1) == S.TRI_SYNC_FREE
    assert S.select_tri(100, 1) == S.TRI_LEVEL_SET
    assert S.select_tri(101, 1) == S.TRI_SYNC_FREE
    assert S.select_tri(20, 15) == S.TRI_LEVEL_SET
    assert S.select_tri(21, 15) == S.TRI_SYNC_FREE
    assert S.select_tri(20, 16) == S.TRI_SYNC_FREE
    assert S.select_tri(2, 2) == S.TRI_LEVEL_SET
    assert S.select_tri(20000, 3) == S.TRI_SYNC_FREE


def test_alg7_square_boundaries():
    S = st
    assert S.select_sq(12, 50, 100) == S.SQ_SCALAR_CSR
    assert S.select_sq(12, 51, 100) == S.SQ_SCALAR_DCSR
    assert S.select_sq(13, 15, 100) == S.SQ_VECTOR_CSR
    assert S.select_sq(13, 16, 100) == S.SQ_VECTOR_DCSR
    assert S.select_sq(0, 7, 7) == S.SQ_SCALAR_DCSR
    # integer comparisons: 3/20 exactly at the boundary
    assert S.select_sq(20, 3, 20) == S.SQ_VECTOR_CSR
    assert S.select_sq(20, 4, 20) == S.SQ_VECTOR_DCSR


# ---------------------------------------------------------- full analysis
def _perm_matrix(M, perm):
    A = _scipy(M)
    P = A[perm][:, perm].tocsr()
    P.sort_indices()
    return P


@pytest.mark.parametrize("variant", ["REC", "COL", "ROW"])
@pytest.mark.parametrize("name", ["C1", "C3", "C4", "C5"])
def test_partition_covers_matrix_and_blocks_solve(variant, name):
    M, b = g.gen_config(name, small=True, nrhs=2)
    A = st.analyse(M, depth=3, variant=variant)
    assert sum(s.nnz for s in A.segs) == M.nnz
    P = _perm_matrix(M, A.perm)
    assert sp.triu(P, 1).nnz == 0  # P L P^T stays lower triangular
    # block execution in the emitted order reproduces Algorithm 1's x
    x_ref = on.solve(M, b)
    w = b[:, A.perm].copy()
    for s in A.segs:
        blk = P[s.row0:s.row1, s.col0:s.col1]
        if s.kind == "SQ":
            w[:, s.row0:s.row1] -= (blk @ w[:, s.col0:s.col1].T).T
        else:
            sub = g.Matrix(n=s.row1 - s.row0, row_ptr=blk.indptr.astype(np.int32),
                           col_idx=blk.indices.astype(np.int32), val=blk.data)
            w[:, s.row0:s.row1] = on.solve(sub, w[:, s.row0:s.row1])
    x = np.empty_like(w)
    x[:, A.perm] = w
    assert on.rel_err(x, x_ref) < 1e-12


def test_reorder_invariants():
    M = g.c3_powerlaw_layers(n=30_011, P=71)
    A0 = st.analyse(M, depth=0)
    A2 = st.analyse(M, depth=2)
    # root reorder of a level-by-level generated matrix is the identity
    assert np.array_equal(A0.perm, np.arange(M.n))
    # leaves are level-sorted (non-decreasing leaf levels)
    for s in A2.segs:
        if s.kind == "TRI":
            lv = A2.leaf_level[s.row0:s.row1]
            assert np.all(np.diff(lv) >= 0)
            assert lv[-1] + 1 == s.nlevels
    # the top child's reorder is the identity: the first quarter of rows keeps
    # the order the root gave it
    q = M.n // 4
    assert np.array_equal(A2.perm[:q], A0.perm[:q])


def test_reorder_stable_closed_form_c2():
    nx, ny = 40, 30
    M = g.c2_laplacian_ic0(nx, ny)
    A = st.analyse(M, depth=0)
    i = np.arange(M.n)
    key = (i % nx) + (i // nx)
    assert np.array_equal(A.perm, np.lexsort((i, key)))  # sort by (ix+iy, i)


def test_c2_full_size_closed_form_blocks():
    """C2 at full size, B200 paper rule: depth 1, top triangle = anti-diagonal
    levels 0..999 (1000 levels), square 1998 nnz with 1000 nonempty rows."""
    M = g.c2_laplacian_ic0(1000)
    A = st.analyse(M, min_block_rows=st.paper_threshold(148 * 128))
    assert A.depth == 1 and len(A.segs) == 3
    top, sq, bot = A.segs
    assert top.nlevels == 1000 and top.row1 == 500_000
    assert sq.nnz == 1998 and sq.empty_rows == 500_000 - 1000
    assert sq.kernel == st.SQ_SCALAR_DCSR
    assert top.kernel == st.TRI_SYNC_FREE and bot.kernel == st.TRI_SYNC_FREE
    assert top.nnz + sq.nnz + bot.nnz == M.nnz


def test_formats_against_scipy():
    M = g.c5_random_multirhs(n=5000)
    A = st.analyse(M, depth=2)
    P = _perm_matrix(M, A.perm)
    for s, arr in zip(A.segs, A.seg_arrays):
        blk = P[s.row0:s.row1, s.col0:s.col1].tocsr()
        rowcounts = np.diff(blk.indptr)
        if s.kind == "TRI":
            assert np.array_equal(arr["IN_DEGREE"], rowcounts - 1)
            assert arr["LEVEL_PTR"][-1] == s.row1 - s.row0
            assert s.nnz_per_row == blk.nnz // (s.row1 - s.row0)
        else:
            assert np.array_equal(arr["DCSR_ROWS"], np.nonzero(rowcounts)[0])
            assert s.empty_rows == int((rowcounts == 0).sum())


def test_upper_via_reversal():
    L = g.c1_random(n=400)
    U = g.to_upper(L)
    A = st.analyse(U, depth=2)
    P = _perm_matrix(U, A.perm)
    assert sp.triu(P, 1).nnz == 0 and P.nnz == U.nnz
    b = g.gen_rhs(U.n, 1, seed=3)
    x_ref = on.solve(U, b)
    Pm = g.Matrix(n=U.n, row_ptr=P.indptr.astype(np.int32), col_idx=P.indices.astype(np.int32),
                  val=P.data)
    xp = on.solve(Pm, b[:, A.perm])
    x = np.empty_like(xp)
    x[:, A.perm] = xp
    assert on.rel_err(x, x_ref) < 1e-13


def test_reorder_none_keeps_identity():
    M, _ = g.gen_config("C5", small=True)
    A = st.analyse(M, depth=2, reorder=False)
    assert np.array_equal(A.perm, np.arange(M.n))
    assert sum(s.nnz for s in A.segs) == M.nnz


def test_clamp_depth_brute_force():
    """R1b by brute force: the clamped depth is the LARGEST d <= the forced
    depth whose REC partition (mid = lo + floor((hi-lo)/2))
    leaves every one of its 2^d triangles non-empty."""
    for n in range(1, 80):
        for forced in range(0, 9):
            ok = [d for d in range(forced + 1)
                  if all(s.row1 > s.row0 for s in st.partition(n, d, "REC") if s.kind == "TRI")]
            assert st.clamp_depth(n, forced) == max(ok), (n, forced)


def test_degenerate_sizes():
    for n in (1, 2, 3):
        M = g.shape_bidiagonal(n)
        A = st.analyse(M, depth=5)
        assert A.depth == st.clamp_depth(n, 5)
        assert sum(s.nnz for s in A.segs) == M.nnz
        assert all(s.row1 > s.row0 for s in A.segs if s.kind == "TRI")
