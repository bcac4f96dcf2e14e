"""CPU tests of the C-ABI library: it loads, exports every symbol that
include/sptrsv.h declares, validates its input, and its host analysis is
bit-exact against the structural oracle (levels, permutation, block
partition, features, Alg 7 labels, formats, the permuted matrix).

No compute call is made here (host_only plans: no device is touched)."""
import ctypes
import os
import re

import numpy as np
import pytest

import paper_conf_icpp_lun020_b200 as sp
from paper_conf_icpp_lun020_b200 import _capi as C
from oracle import structure as st
from workloads import generators as g

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
B200_T = 20 * 148 * 128


@pytest.fixture(scope="module", autouse=True)
def _built():
    from paper_conf_icpp_lun020_b200 import build
    build.build()


def test_exports_every_declared_symbol():
    hdr = open(os.path.join(ROOT, "include", "sptrsv.h")).read()
    hdr = re.sub(r"/\*.*?\*/", "", hdr, flags=re.S)  # drop comments
    declared = set(re.findall(r"\b(sptrsv_[a-z_]+)\s*\(", hdr))
    assert {"sptrsv_analyse", "sptrsv_solve", "sptrsv_free"} <= declared
    L = C.lib()
    for name in declared:
        assert hasattr(L, name), name
    assert declared == set(C.EXPORTS)
    assert "sm_100a" in sp.version()


def _analyse(M, **kw):
    kw.setdefault("host_only", True)
    kw.setdefault("reorder", True)  # the paper's level-set reordering (L231); "auto" is tested below
    kw.setdefault("min_block_rows", B200_T)
    return sp.sptrsv_analyse(M.row_ptr, M.col_idx, M.val, fill=M.uplo, **kw)


def _compare(M, plan, A):
    info = plan.info()
    assert info["n"] == M.n and info["nnz"] == M.nnz and info["depth"] == A.depth
    assert np.array_equal(plan.perm(), A.perm)
    assert np.array_equal(plan.levels(), A.leaf_level)
    segs = plan.segments()
    assert len(segs) == len(A.segs)
    for i, (s, o) in enumerate(zip(segs, A.segs)):
        got = (s["kind"], s["row0"], s["row1"], s["col0"], s["col1"], s["nnz"], s["nlevels"],
               s["nnz_per_row"], s["empty_rows"], s["kernel"], s["format"])
        want = (o.kind, o.row0, o.row1, o.col0, o.col1, o.nnz, o.nlevels, o.nnz_per_row, o.empty_rows,
                o.kernel, o.format)
        assert got == want, (i, got, want)
        arrs = A.seg_arrays[i]
        if o.kind == "TRI":
            assert np.array_equal(plan.seg_array(i, C.ARRAY_IN_DEGREE), arrs["IN_DEGREE"])
            assert np.array_equal(plan.seg_array(i, C.ARRAY_LEVEL_PTR), arrs["LEVEL_PTR"])
        else:
            assert np.array_equal(plan.seg_array(i, C.ARRAY_DCSR_ROWS), arrs["DCSR_ROWS"])
    rp, ci, va = plan.matrix()
    assert np.array_equal(rp, A.p_row_ptr)
    assert np.array_equal(ci, A.p_col_idx)
    assert np.array_equal(va.view(np.uint8), np.asarray(A.p_val, dtype=va.dtype).view(np.uint8))


@pytest.mark.parametrize("name", ["C1", "C2", "C3", "C4", "C5"])
@pytest.mark.parametrize("variant", ["REC", "COL", "ROW"])
@pytest.mark.parametrize("depth", [0, 2, 3])
def test_structure_parity_small_configs(name, variant, depth):
    M, _ = g.gen_config(name, small=True)
    plan = _analyse(M, variant=variant, depth=depth)
    A = st.analyse(M, depth=depth, variant=variant)
    _compare(M, plan, A)


@pytest.mark.parametrize("name", ["C1", "C3", "C5"])
def test_structure_parity_upper(name):
    M, _ = g.gen_config(name, small=True)
    U = g.to_upper(M)
    plan = _analyse(U, depth=2)
    _compare(U, plan, st.analyse(U, depth=2))


@pytest.mark.parametrize("name", ["C1", "C2", "C3", "C5"])
@pytest.mark.parametrize("uplo", ["L", "U"])
def test_structure_parity_transpose(name, uplo):
    """transpose=1 (R31): the plan of A analysed for A^T x = b is, bit for bit,
    the oracle's analysis of A^T (the other fill), for both fills of A."""
    M, _ = g.gen_config(name, small=True)
    if uplo == "U":
        M = g.to_upper(M)
    plan = _analyse(M, depth=2, transpose=True)
    MT = g.transpose(M)
    assert plan.info()["fill"] == (C.UPPER if uplo == "L" else C.LOWER)
    _compare(MT, plan, st.analyse(MT, depth=2))


def test_transpose_large_matches_analysed_transpose():
    """Above the parallel grain: the library's host transpose gives the same
    plan as analysing the explicitly transposed input (plan hash, perm,
    segments and P A P^T bit for bit)."""
    M = g.c5_random_multirhs(n=150_001)
    a = _analyse(M, depth=3, transpose=True, threads=16)
    MT = g.transpose(M)
    b = _analyse(MT, depth=3, threads=16)
    assert a.hash() == b.hash()
    assert np.array_equal(a.perm(), b.perm())
    assert a.segments() == b.segments()
    for x, y in zip(a.matrix(), b.matrix()):
        assert np.array_equal(x, y)


@pytest.mark.parametrize("name", ["C3", "C4"])
def test_structure_parity_no_reorder(name):
    M, _ = g.gen_config(name, small=True)
    plan = _analyse(M, depth=2, reorder=False)
    _compare(M, plan, st.analyse(M, depth=2, reorder=False))


def test_structure_parity_paper_rule_and_threshold():
    M, _ = g.gen_config("C3", small=True)
    for T in (5000, 7000, 20000, 10 ** 9):
        plan = _analyse(M, min_block_rows=T)
        _compare(M, plan, st.analyse(M, min_block_rows=T))


def test_structure_parity_c2_full_size():
    M, _ = g.gen_config("C2")
    plan = _analyse(M)
    A = st.analyse(M, min_block_rows=B200_T)
    _compare(M, plan, A)
    assert plan.info()["depth"] == 1


def test_b200_depth_retune_keeps_narrow_root_whole():
    """Reading R30: with the library's defaults (selector B200, depth and
    min_block_rows unset) a 2-D stencil IC(0) root -- every level <= 2,048
    rows, <= 2 dependencies per row -- stays one triangle (the wavefront
    solves it whole); the structure is then the oracle's at depth 0.  On a
    4M-row grid the B200 threshold (R33) alone would still split once, so
    R30 is what keeps it whole.  An explicit min_block_rows (or depth)
    restores the paper's rule; so does PAPER."""
    M = g.c2_laplacian_ic0(2000)  # n = 4M: R33's T (1.5M rows) gives depth 1
    plan = sp.sptrsv_analyse(M.row_ptr, M.col_idx, M.val, host_only=True)
    info = plan.info()
    assert info["depth"] == 0 and info["depth_rule"] == 1
    assert [s["impl"] for s in plan.segments()] == ["TRI_PIPE"]
    paper = sp.sptrsv_analyse(M.row_ptr, M.col_idx, M.val, host_only=True, selector="PAPER")
    assert paper.info()["depth"] == 3 and paper.info()["depth_rule"] == 0
    M, _ = g.gen_config("C2")
    plan = sp.sptrsv_analyse(M.row_ptr, M.col_idx, M.val, host_only=True)
    assert plan.info()["depth"] == 0 and plan.info()["depth_rule"] in (1, 3)
    _compare(M, plan, st.analyse(M, depth=0))
    paper = sp.sptrsv_analyse(M.row_ptr, M.col_idx, M.val, host_only=True, selector="PAPER")
    assert paper.info()["depth"] == 1 and paper.info()["depth_rule"] == 0
    forced = sp.sptrsv_analyse(M.row_ptr, M.col_idx, M.val, host_only=True, depth=1)
    assert forced.info()["depth_rule"] == 2
    # a wide-level root keeps the paper's depth (C5 shape, 150K rows: 0 either way)
    M5 = g.c5_random_multirhs(n=150_001)
    p5 = sp.sptrsv_analyse(M5.row_ptr, M5.col_idx, M5.val, host_only=True)
    assert p5.info()["depth_rule"] == 0


def test_b200_depth_threshold_r33():
    """Reading R33: under the B200 selector with depth / min_block_rows unset,
    the L299 threshold is 4 x 20 x SMs x 128; a C5-shaped root of 800K rows
    (paper: depth 1) stays whole, reported as depth_rule 3, and its structure
    is the oracle's at that depth; the PAPER selector and an explicit
    min_block_rows keep the paper's threshold."""
    M = g.c5_random_multirhs(n=800_000)
    plan = sp.sptrsv_analyse(M.row_ptr, M.col_idx, M.val, host_only=True)
    info = plan.info()
    T = 20 * info["sm_count"] * 128
    assert info["min_block_rows"] == 4 * T
    assert info["depth"] == st.depth_rule(M.n, 4 * T) == 0 and info["depth_rule"] == 3
    _compare(M, plan, st.analyse(M, depth=0))
    paper = sp.sptrsv_analyse(M.row_ptr, M.col_idx, M.val, host_only=True, selector="PAPER")
    assert paper.info()["depth"] == st.depth_rule(M.n, T) == 1 and paper.info()["depth_rule"] == 0
    explicit = sp.sptrsv_analyse(M.row_ptr, M.col_idx, M.val, host_only=True, min_block_rows=T)
    assert explicit.info()["depth"] == 1 and explicit.info()["depth_rule"] == 0


@pytest.mark.parametrize("shape", ["diag", "chain", "dense", "arrow", "fig1", "n1", "n2", "empty"])
def test_structure_parity_adversarial(shape):
    M = {"diag": lambda: g.shape_diagonal(1000), "chain": lambda: g.shape_bidiagonal(3000),
         "dense": lambda: g.shape_dense_lower(150), "arrow": lambda: g.shape_arrow(999),
         "fig1": g.shape_paper_fig1, "n1": lambda: g.shape_diagonal(1),
         "n2": lambda: g.shape_bidiagonal(2), "empty": lambda: g.shape_diagonal(0)}[shape]()
    for depth in (0, 1, 4):
        plan = _analyse(M, depth=depth)
        _compare(M, plan, st.analyse(M, depth=depth))


def test_deterministic_across_thread_counts():
    M, _ = g.gen_config("C5", small=True)
    a = _analyse(M, depth=3, threads=1)
    b = _analyse(M, depth=3, threads=7)
    assert np.array_equal(a.perm(), b.perm())
    assert a.segments() == b.segments()
    for x, y in zip(a.matrix(), b.matrix()):
        assert np.array_equal(x, y)


@pytest.mark.parametrize("uplo", ["L", "U"])
def test_deterministic_across_thread_counts_large(uplo):
    """n above the parallel grain (65,536 rows): the parallel validation,
    J U J mapping, P L P^T, bottom-child reorders and segment extraction (per
    segment with few threads, per row with many) give the same plan, bit for
    bit, as one thread -- the replicated multi-GPU plan relies on it."""
    M = g.c5_random_multirhs(n=150_001)
    if uplo == "U":
        M = g.to_upper(M)
    plans = [_analyse(M, depth=3, threads=t) for t in (1, 5, 16)]
    h = [p.hash() for p in plans]
    assert h[0] == h[1] == h[2]
    for p in plans[1:]:
        assert np.array_equal(plans[0].perm(), p.perm())
        assert plans[0].segments() == p.segments()
        for x, y in zip(plans[0].matrix(), p.matrix()):
            assert np.array_equal(x, y)
    _compare(M, plans[1], st.analyse(M, depth=3))


# ------------------------------------------------------------ validation
def _expect(status, rp, ci, val, fill="L", **kw):
    with pytest.raises(sp.SptrsvError) as e:
        sp.sptrsv_analyse(np.array(rp), np.array(ci), np.array(val, dtype=np.float64), fill=fill,
                          host_only=True, **kw)
    assert e.value.status_name == status, str(e.value)


def test_validation_errors():
    _expect("UNSORTED", [0, 1, 3], [0, 1, 0], [1.0, 1.0, 1.0])          # row 1 cols 1,0
    _expect("UNSORTED", [0, 1, 3], [0, 0, 0], [1.0, 1.0, 1.0])          # duplicate
    _expect("NOT_TRIANGULAR", [0, 2, 3], [0, 1, 1], [1.0, 2.0, 1.0])    # (0,1) above diag
    _expect("ZERO_PIVOT", [0, 1, 2], [0, 0], [1.0, 2.0])                # row 1 has no diagonal
    _expect("ZERO_PIVOT", [0, 1, 3], [0, 0, 1], [1.0, 2.0, 0.0])        # zero diagonal
    _expect("NOT_TRIANGULAR", [0, 1, 3], [0, 0, 1], [1.0, 2.0, 1.0], fill="U")  # (1,0) below diag
    _expect("INVALID_VALUE", [0, 1, 3], [0, 0, 5], [1.0, 2.0, 1.0])     # column out of range
    _expect("INVALID_VALUE", [1, 1, 3], [0, 0, 1], [1.0, 2.0, 1.0])     # row_ptr[0] != 0


def test_transpose_validates_the_given_fill():
    """transpose=1 (R31) checks A with its own fill before transposing: an
    entry above the diagonal of a LOWER input is still NOT_TRIANGULAR, a
    missing diagonal still ZERO_PIVOT; a bad transpose value is rejected."""
    _expect("NOT_TRIANGULAR", [0, 2, 3], [0, 1, 1], [1.0, 2.0, 1.0], transpose=True)
    _expect("ZERO_PIVOT", [0, 1, 2], [0, 0], [1.0, 2.0], transpose=True)
    _expect("NOT_TRIANGULAR", [0, 1, 3], [0, 0, 1], [1.0, 2.0, 1.0], fill="U", transpose=True)
    o = C.Opts()
    C.lib().sptrsv_opts_default(ctypes.byref(o))
    assert o.transpose == 0
    o.transpose = 2
    o.host_only = 1
    rp = np.array([0, 1], dtype=np.int32)
    ci = np.array([0], dtype=np.int32)
    va = np.array([1.0])
    h = ctypes.c_void_p()
    st_ = C.lib().sptrsv_analyse(1, 1, rp.ctypes.data_as(ctypes.c_void_p), ci.ctypes.data_as(ctypes.c_void_p),
                                 va.ctypes.data_as(ctypes.c_void_p), 0, C.LOWER, ctypes.byref(o), None,
                                 ctypes.byref(h))
    assert st_ == 1 and not h.value  # SPTRSV_ERROR_INVALID_VALUE, no plan


def test_validation_error_names_row():
    with pytest.raises(sp.SptrsvError) as e:
        sp.sptrsv_analyse(np.array([0, 1, 2, 4]), np.array([0, 1, 0, 1]), np.ones(4), host_only=True)
    assert "row 2" in str(e.value)


@pytest.mark.parametrize("threads", [1, 16])
def test_validation_reports_lowest_bad_row_in_parallel(threads):
    """Rows are validated in parallel chunks; the error is still the one a
    serial row-order scan meets first (the lowest bad row)."""
    M = g.c5_random_multirhs(n=150_001)
    ci, val = M.col_idx.copy(), M.val.copy()
    r_zero, r_unsorted = 120_003, 100_001  # zero pivot late, unsorted earlier
    val[M.row_ptr[r_zero + 1] - 1] = 0.0
    a = M.row_ptr[r_unsorted]
    ci[a], ci[a + 1] = ci[a + 1], ci[a]
    with pytest.raises(sp.SptrsvError) as e:
        sp.sptrsv_analyse(M.row_ptr, ci, val, host_only=True, threads=threads)
    assert e.value.status_name == "UNSORTED" and f"row {r_unsorted}" in str(e.value)
    ci2 = M.col_idx.copy()
    with pytest.raises(sp.SptrsvError) as e:
        sp.sptrsv_analyse(M.row_ptr, ci2, val, host_only=True, threads=threads)
    assert e.value.status_name == "ZERO_PIVOT" and f"row {r_zero}" in str(e.value)


def test_float32_plan_structure_matches_float64():
    M, _ = g.gen_config("C4", small=True)
    a = _analyse(M, depth=2)
    b = _analyse(M.astype(np.float32), depth=2)
    assert np.array_equal(a.perm(), b.perm())
    assert a.segments() == b.segments()


def test_host_only_plan_refuses_solve():
    M = g.shape_diagonal(4)
    plan = _analyse(M)
    with pytest.raises(sp.SptrsvError) as e:
        plan.solve(np.ones(4))
    assert e.value.status_name == "NOT_SUPPORTED"


@pytest.mark.parametrize("name,expect_none", [("C1", False), ("C2", False), ("C3", False), ("C4", True),
                                              ("C5", False)])
def test_reorder_auto_keeps_supernodal_inputs(name, expect_none):
    """reorder="auto" (R29) skips the level sort only for supernodal
    inputs; whatever it picks, the structure equals the oracle's for that
    choice."""
    M, _ = g.gen_config(name, small=True)
    plan = _analyse(M, depth=2, reorder="auto")
    eff_none = plan.info()["reorder"] == 1
    assert eff_none == expect_none
    _compare(M, plan, st.analyse(M, depth=2, reorder=not eff_none))


def test_supernode_pieces_cover_dense_blocks():
    """The supernodal selector only fires on triangles made of dense diagonal
    blocks: the C4 factor (64-wide supernodes -> 32-row pieces), the dense
    lower triangle; never on a bidiagonal chain (its diagonal blocks are not
    dense) or on C2/C3."""
    for M, want in [(g.gen_config("C4", small=True)[0], True), (g.shape_dense_lower(150), True),
                    (g.shape_bidiagonal(3000), False), (g.gen_config("C2", small=True)[0], False),
                    (g.gen_config("C3", small=True)[0], False)]:
        plan = _analyse(M, depth=0, reorder="auto")
        seg = plan.segments()[0]
        assert (seg["impl"] == "TRI_SUPERNODE") == want, (M.name, seg["impl"])
