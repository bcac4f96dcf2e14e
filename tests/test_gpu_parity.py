"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle.

Bars (BASELINE.json north_star): fp64 rel_err <= 1e-10,
fp32 rel_err <= 1e-4 against the fp64 oracle on the fp64 data; every fp64
result also satisfies the componentwise backward-error bound of substitution
(oracle.numeric.residual_bound_ok), which holds for any summation order.
"""
import numpy as np
import pytest
import torch

import paper_conf_icpp_lun020_b200 as sp
from oracle import numeric as on
from oracle import structure as st
from workloads import generators as g

pytestmark = pytest.mark.gpu
TOL64, TOL32 = 1e-10, 1e-4
B200_T = 20 * 148 * 128


def _solve(M, b, dtype=torch.float64, layout="col", **kw):
    """b: numpy (nrhs, n).  Returns x numpy (nrhs, n) float64."""
    val = M.val if dtype == torch.float64 else M.val.astype(np.float32)
    plan = sp.sptrsv_analyse(M.row_ptr, M.col_idx, val, fill=M.uplo, **kw)
    bt = torch.from_numpy(b).to("cuda", dtype)
    if layout == "col":
        B = bt.T  # (n, nrhs) column-major
    else:
        B = bt.T.contiguous()  # (n, nrhs) row-major
    if b.shape[0] == 1:
        B = bt[0].contiguous()
    X = sp.sptrsv_solve(plan, B)
    torch.cuda.synchronize()
    x = X.double().cpu().numpy()
    x = x[None] if x.ndim == 1 else x.T
    return x, plan


def _check64(M, b, x):
    ref = on.solve(M, b)
    err = on.rel_err(x, ref)
    assert err <= TOL64, err
    ok, worst = on.residual_bound_ok(M, x, b)
    assert ok, worst
    return err


CONFIGS = ["C1", "C2", "C3", "C4", "C5"]


@pytest.mark.parametrize("name", CONFIGS)
@pytest.mark.parametrize("selector", ["PAPER", "B200"])
def test_small_configs_default(gpu, name, selector):
    M, b = g.gen_config(name, small=True, nrhs=1)
    x, _ = _solve(M, b, selector=selector, min_block_rows=max(2, M.n // 9))
    _check64(M, b, x)


@pytest.mark.parametrize("name", CONFIGS)
@pytest.mark.parametrize("tri", ["TRI_LEVELSET", "TRI_SYNCFREE", "TRI_CHAIN", "TRI_SUPERNODE", "TRI_PIPE"])
@pytest.mark.parametrize("sq", ["SQ_SCALAR", "SQ_VECTOR", "SQ_ADAPT"])
def test_forced_kernels(gpu, name, tri, sq):
    M, b = g.gen_config(name, small=True, nrhs=1)
    if tri == "TRI_LEVELSET" and name in ("C2",):
        pytest.skip("thousands of per-level launches; covered by C1/C3-C5")
    x, plan = _solve(M, b, depth=2, force_tri_impl=tri, force_sq_impl=sq, reorder=True)
    # the wavefront hands rows with > 8 dependencies to the chain kernel
    ok = (tri, "TRI_CHAIN") if tri == "TRI_PIPE" and name in ("C3", "C4", "C5") else (tri,)
    assert all(s["impl"] in ok for s in plan.segments() if s["kind"] == "TRI" and s["nlevels"] > 1)
    _check64(M, b, x)


@pytest.mark.parametrize("name", CONFIGS)
@pytest.mark.parametrize("variant", ["REC", "COL", "ROW"])
def test_variants(gpu, name, variant):
    M, b = g.gen_config(name, small=True, nrhs=1)
    x, _ = _solve(M, b, depth=3, variant=variant)
    _check64(M, b, x)


@pytest.mark.parametrize("name", CONFIGS)
@pytest.mark.parametrize("nrhs", [2, 7, 33, 70])
@pytest.mark.parametrize("tri", ["TRI_LEVELSET", "TRI_SYNCFREE", "TRI_CHAIN", "TRI_SUPERNODE", "TRI_PIPE"])
def test_multi_rhs(gpu, name, nrhs, tri):
    if tri == "TRI_LEVELSET" and name == "C2":
        pytest.skip("per-level launches")
    M, b = g.gen_config(name, small=True, nrhs=nrhs)
    x, _ = _solve(M, b, depth=2, force_tri_impl=tri, reorder=True)
    _check64(M, b, x)


@pytest.mark.parametrize("tri", ["TRI_LEVELSET", "TRI_CHAIN", "TRI_SYNCFREE", "TRI_SUPERNODE", "TRI_PIPE"])
def test_no_reorder_never_walks_levels(gpu, tri):
    """Without the level-set reordering, levels are not contiguous row
    ranges: a forced level-set / chain kernel falls back to sync-free."""
    M, b = g.gen_config("C3", small=True, nrhs=1)
    x, plan = _solve(M, b, depth=2, force_tri_impl=tri, reorder=False)
    assert all(s["impl"] in ("TRI_SYNCFREE", "TRI_SUPERNODE", "TRI_DIAG") for s in plan.segments()
               if s["kind"] == "TRI")
    _check64(M, b, x)


@pytest.mark.parametrize("name", ["C4", "C1"])
@pytest.mark.parametrize("reorder", ["auto", True, False])
def test_supernodal_default_and_reorders(gpu, name, reorder):
    """C4 (supernodal) under the B200 default picks reorder=none + the
    supernodal kernel; every reorder choice solves to the oracle."""
    M, b = g.gen_config(name, small=True, nrhs=1)
    x, plan = _solve(M, b, depth=1, reorder=reorder)
    if name == "C4" and reorder != True:  # noqa: E712
        assert any(s["impl"] == "TRI_SUPERNODE" for s in plan.segments())
    _check64(M, b, x)


@pytest.mark.parametrize("nrhs", [15, 16, 64, 65, 130])
@pytest.mark.parametrize("dtype", [torch.float64, torch.float32])
@pytest.mark.parametrize("layout", ["col", "row"])
def test_supernode_multi_rhs(gpu, nrhs, dtype, layout):
    """f-3: C4's supernodal plan with nrhs >= 16 runs tri_supernode_multi
    (64-column chunks, ragged last chunk at 65 / 130, ragged 32-row pieces);
    15 RHS take the sync-free SpTRSM kernel."""
    M, b = g.gen_config("C4", small=True, nrhs=nrhs)
    x, plan = _solve(M, b, dtype=dtype, layout=layout, depth=1)
    assert any(s["impl"] == "TRI_SUPERNODE" for s in plan.segments())
    if dtype == torch.float64:
        _check64(M, b, x)
    else:
        assert on.rel_err(x, on.solve(M, b)) <= TOL32


def test_supernode_multi_repeated_solves_epochs(gpu):
    """A multi-RHS solve owns one epoch per 64-column chunk (one supernodal
    launch per chunk): repeated solves on one plan with changing RHS counts
    never see a stale flag."""
    M, b = g.gen_config("C4", small=True, nrhs=130)
    plan = sp.sptrsv_analyse(M.row_ptr, M.col_idx, M.val, depth=1)
    for k in (130, 20, 130, 64, 3, 130):
        bk = np.ascontiguousarray(b[:k]) * (1.0 + 0.1 * k)
        X = sp.sptrsv_solve(plan, torch.from_numpy(bk).cuda().T)
        torch.cuda.synchronize()
        _check64(M, bk, X.T.cpu().numpy())
    plan.free()


def _host_threads():
    import os
    return max(1, len(os.sched_getaffinity(0)))


def test_full_size_c4_supernode_multi_all_columns(gpu):
    """C4 at full size (n=500K, 80M nnz) with 64 RHS through the default
    plan: EVERY column against the oracle (rel_err), the componentwise
    backward-error bound on every 4th column (its extended-precision residual
    costs ~1 s per column on the host)."""
    M, b = g.gen_config("C4", nrhs=64)
    plan = sp.sptrsv_analyse(M.row_ptr, M.col_idx, M.val)
    X = sp.sptrsv_solve(plan, torch.from_numpy(b).cuda().T)
    torch.cuda.synchronize()
    xs = X.T.cpu().numpy()
    ref = on.solve(M, b, threads=_host_threads())
    errs = [on.rel_err(xs[c], ref[c]) for c in range(64)]
    assert max(errs) <= TOL64, (int(np.argmax(errs)), max(errs))
    cols = list(range(0, 64, 4)) + [63]
    ok, worst = on.residual_bound_ok(M, xs[cols], b[cols])
    assert ok, worst


@pytest.mark.parametrize("layout", ["col", "row"])
def test_layouts(gpu, layout):
    M, b = g.gen_config("C5", small=True, nrhs=9)
    x, _ = _solve(M, b, layout=layout, depth=2)
    _check64(M, b, x)


@pytest.mark.parametrize("name", CONFIGS)
def test_fp32(gpu, name):
    M, b = g.gen_config(name, small=True, nrhs=1)
    x, _ = _solve(M, b, dtype=torch.float32, depth=2)
    assert on.rel_err(x, on.solve(M, b)) <= TOL32


@pytest.mark.parametrize("name", ["C1", "C3", "C5"])
def test_upper(gpu, name):
    M, b = g.gen_config(name, small=True, nrhs=2)
    U = g.to_upper(M)
    x, _ = _solve(U, b, depth=2)
    _check64(U, b, x)


@pytest.mark.parametrize("name", CONFIGS)
@pytest.mark.parametrize("uplo", ["L", "U"])
@pytest.mark.parametrize("nrhs", [1, 5])
def test_transpose(gpu, name, uplo, nrhs):
    """transpose=1 (R31): the plan of A solves A^T x = b; the oracle solves
    the explicitly transposed input."""
    M, b = g.gen_config(name, small=True, nrhs=nrhs)
    if uplo == "U":
        M = g.to_upper(M)
    x, _ = _solve(M, b, depth=2, transpose=True)
    _check64(g.transpose(M), b, x)


@pytest.mark.parametrize("name", ["C2", "C3", "C4"])
def test_full_size_transpose(gpu, name):
    """Full BASELINE sizes, default options: L^T x = b (the backward sweep of
    an IC(0) / supernodal preconditioner application)."""
    M, b = g.gen_config(name, nrhs=1)
    x, plan = _solve(M, b, transpose=True)
    _check64(g.transpose(M), b, x)


def test_ic0_pcg_driver(gpu):
    """f-4: the preconditioner application L^-T L^-1 r through the forward and
    transposed plans matches the oracle's two substitutions, and IC(0)-PCG on
    the 5-point Laplacian converges in fewer iterations than CG."""
    import importlib.util, os
    spec = importlib.util.spec_from_file_location(
        "ic0_pcg", os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "examples", "ic0_pcg.py"))
    ex = importlib.util.module_from_spec(spec)
    spec.loader.exec_module(ex)
    nx = 120
    L = g.c2_laplacian_ic0(nx)
    M = ex.IC0(L)
    r = g.gen_rhs(L.n, 1, seed=5)[0]
    z = M(torch.from_numpy(r).cuda()).cpu().numpy()
    ref = on.solve(g.transpose(L), on.solve(L, r))
    assert on.rel_err(z[None], ref[None]) <= TOL64
    Ms = ex.IC0(L, same_plan=True)  # the L^-T sweep from the forward plan (R32)
    zs = Ms(torch.from_numpy(r).cuda()).cpu().numpy()
    assert on.rel_err(zs[None], ref[None]) <= TOL64
    Ms.free()
    A = ex.laplacian_csr(nx, nx, torch.device("cuda"))
    b = torch.from_numpy(g.gen_rhs(L.n, 1, seed=6)[0]).cuda()
    x0, it_cg, h0 = ex.pcg(A, b, None, 1e-10)
    x1, it_pcg, h1 = ex.pcg(A, b, M, 1e-10)
    M.free()
    assert h0[-1] <= 1e-10 and h1[-1] <= 1e-10
    assert it_pcg < it_cg, (it_pcg, it_cg)
    assert float(torch.linalg.vector_norm(x0 - x1) / torch.linalg.vector_norm(x0)) < 1e-8


def test_repeated_solves_epoch(gpu):
    M, b = g.gen_config("C3", small=True, nrhs=1)
    plan = sp.sptrsv_analyse(M.row_ptr, M.col_idx, M.val, depth=2, force_tri_impl="TRI_SYNCFREE")
    B = torch.from_numpy(b[0]).cuda()
    ref = on.solve(M, b)
    for _ in range(20):
        X = plan.solve(B)
    torch.cuda.synchronize()
    assert on.rel_err(X.cpu().numpy()[None], ref) <= TOL64


def test_in_place(gpu):
    M, b = g.gen_config("C5", small=True, nrhs=4)
    plan = sp.sptrsv_analyse(M.row_ptr, M.col_idx, M.val, depth=2)
    B = torch.from_numpy(b).cuda().T
    sp.sptrsv_solve(plan, B, x=B)
    torch.cuda.synchronize()
    _check64(M, b, B.T.cpu().numpy())


def test_host_pointers(gpu):
    M, b = g.gen_config("C2", small=True, nrhs=3)
    plan = sp.sptrsv_analyse(M.row_ptr, M.col_idx, M.val)
    Bh = np.ascontiguousarray(b.T)  # (n, 3) row-major host
    X = sp.sptrsv_solve(plan, Bh)
    _check64(M, b, X.T)
    Bp = torch.from_numpy(b).pin_memory().T  # pinned host, column-major
    Xp = sp.sptrsv_solve(plan, Bp)
    _check64(M, b, Xp.T.numpy())


@pytest.mark.parametrize("nrhs", [32, 37, 133])
@pytest.mark.parametrize("pinned", [True, False])
def test_host_pointers_pipelined(gpu, nrhs, pinned):
    """Host buffers with >= 32 column-major RHS go through the column-block
    pipeline (copy in / solve / copy out overlapped on three streams), with
    ragged last blocks and ld > n."""
    M, b = g.gen_config("C5", small=True, nrhs=nrhs)
    plan = sp.sptrsv_analyse(M.row_ptr, M.col_idx, M.val, depth=2)
    n = M.n
    big = torch.zeros((nrhs, n + 5), dtype=torch.float64)
    big[:, :n] = torch.from_numpy(b)
    if pinned:
        big = big.pin_memory()
    B = big[:, :n].T  # (n, nrhs) column-major, ld = n + 5
    X = torch.full((nrhs, n + 3), float("nan"), dtype=torch.float64)
    if pinned:
        X = X.pin_memory()
    Xv = X[:, :n].T
    sp.sptrsv_solve(plan, B, Xv)
    _check64(M, b, X[:, :n].numpy())
    assert torch.isnan(X[:, n:]).all()  # the ld padding is untouched


@pytest.mark.parametrize("shape", ["diag", "chain", "dense", "arrow", "n1", "fig1"])
def test_adversarial(gpu, shape):
    M = {"diag": lambda: g.shape_diagonal(10000), "chain": lambda: g.shape_bidiagonal(100_000),
         "dense": lambda: g.shape_dense_lower(300), "arrow": lambda: g.shape_arrow(5000),
         "n1": lambda: g.shape_diagonal(1), "fig1": g.shape_paper_fig1}[shape]()
    b = g.gen_rhs(M.n, 1, seed=5)
    for tri in (None, "TRI_SYNCFREE", "TRI_CHAIN"):
        x, _ = _solve(M, b, depth=1 if M.n > 1 else 0, force_tri_impl=tri)
        _check64(M, b, x)


def test_long_chain_near_serial(gpu):
    # nlevels > 20000 -> NEAR_SERIAL label (Alg 7), single-CTA chain kernel
    M = g.shape_bidiagonal(300_000)
    b = g.gen_rhs(M.n, 1, seed=6)
    x, plan = _solve(M, b, selector="PAPER")
    segs = plan.segments()
    assert segs[0]["kernel"] == "NEAR_SERIAL" and segs[0]["impl"] == "TRI_CHAIN"
    _check64(M, b, x)


def test_zero_rhs_and_empty(gpu):
    M = g.shape_diagonal(10)
    plan = sp.sptrsv_analyse(M.row_ptr, M.col_idx, M.val)
    B = torch.zeros(10, 0, dtype=torch.float64, device="cuda")
    sp.sptrsv_solve(plan, B)
    E = g.shape_diagonal(0)
    pe = sp.sptrsv_analyse(E.row_ptr, E.col_idx, E.val)
    sp.sptrsv_solve(pe, torch.zeros(0, dtype=torch.float64, device="cuda"))


def test_mixed_pointers_rejected(gpu):
    M = g.shape_diagonal(10)
    plan = sp.sptrsv_analyse(M.row_ptr, M.col_idx, M.val)
    with pytest.raises(sp.SptrsvError):
        sp.sptrsv_solve(plan, torch.ones(10, dtype=torch.float64, device="cuda"), x=np.zeros(10))


# ------------------------------------------------------------- full sizes
@pytest.mark.parametrize("name", ["C1", "C2", "C3", "C4"])
def test_full_size_configs(gpu, name):
    """BASELINE.json sizes, default options (what bench.py times)."""
    M, b = g.gen_config(name, nrhs=1)
    x, plan = _solve(M, b)
    err = _check64(M, b, x)
    # the plan's structure at full size is the oracle's (for the reorder the
    # B200 default chose: none for the supernodal C4, level otherwise, R29)
    # at the depth the plan reports (the B200 depth retune keeps C2 whole, R30)
    A = st.analyse(M, depth=plan.info()["depth"], reorder=plan.info()["reorder"] == 0)
    segs = plan.segments()
    assert [(s["row0"], s["row1"], s["col0"], s["col1"], s["nnz"], s["nlevels"], s["kernel"])
            for s in segs] == [(o.row0, o.row1, o.col0, o.col1, o.nnz, o.nlevels, o.kernel) for o in A.segs]
    assert np.array_equal(plan.perm(), A.perm)
    print(name, "rel_err", err)


def test_full_size_c5_multi_rhs_all_columns(gpu):
    """C5: n=2M, 512 RHS in one solve (the RPT=16 lane layout of the SpTRSM
    kernels is reached only at nrhs > 256): EVERY column against the oracle
    (rel_err), the backward-error bound on every 16th column and the last."""
    M, b = g.gen_config("C5", nrhs=512)
    plan = sp.sptrsv_analyse(M.row_ptr, M.col_idx, M.val)
    B = torch.from_numpy(b).cuda().T
    X = sp.sptrsv_solve(plan, B)
    torch.cuda.synchronize()
    xs = X.T.cpu().numpy()
    del X, B
    ref = on.solve(M, b, threads=_host_threads())
    errs = [on.rel_err(xs[c], ref[c]) for c in range(512)]
    assert max(errs) <= TOL64, (int(np.argmax(errs)), max(errs))
    cols = list(range(0, 512, 16)) + [511]
    ok, worst = on.residual_bound_ok(M, xs[cols], b[cols])
    assert ok, worst


@pytest.mark.parametrize("geom", ["1,1,1,2", "1,4,2,2", "3,3,2,3", "8,4,8,4", "16,2,8,3"])
@pytest.mark.parametrize("dtype", [torch.float64, torch.float32])
def test_wave_geometries(gpu, geom, dtype, monkeypatch):
    """The strand wavefront at several cluster geometries (SPTRSV_WAVE =
    CTAs,warps,groups-per-chunk,ring-depth): one strand, one CTA, odd
    shapes, the default 8x4 and a non-portable 16-CTA cluster."""
    monkeypatch.setenv("SPTRSV_WAVE", geom)
    for name in ("C2", "C5", "C1"):
        M, b = g.gen_config(name, small=True, nrhs=1)
        x, plan = _solve(M, b, dtype=dtype, depth=1, force_tri_impl="TRI_PIPE", reorder=True)
        if name != "C5":  # C5 rows have up to 9 dependencies: the chain kernel takes them
            assert all(s["impl"] == "TRI_PIPE" for s in plan.segments() if s["kind"] == "TRI" and s["nlevels"] > 1)
        if dtype == torch.float64:
            _check64(M, b, x)
        else:
            assert on.rel_err(x, on.solve(M, b)) <= TOL32


@pytest.mark.parametrize("hook", [("SPTRSV_WAVE_XW", "64"), ("SPTRSV_WAVE_ICAP", "0"), ("SPTRSV_WAVE_ICAP", "5")])
def test_wave_global_fallbacks(gpu, hook, monkeypatch):
    """Own-window and import-capacity overflow: those dependencies are polled
    in global memory (value-as-flag) instead of shared memory."""
    monkeypatch.setenv(*hook)
    for name in ("C2", "C5"):
        M, b = g.gen_config(name, small=True, nrhs=1)
        x, plan = _solve(M, b, depth=1, force_tri_impl="TRI_PIPE", reorder=True)
        _check64(M, b, x)


def test_wave_is_the_c2_default(gpu):
    """C2 (2D stencil IC(0), narrow anti-diagonal levels) runs its triangles on
    the wavefront by default, and nrhs > 1 on the same plan solves too."""
    M, b = g.gen_config("C2", small=True, nrhs=3)
    x, plan = _solve(M, b[:1], depth=1)
    assert [s["impl"] for s in plan.segments() if s["kind"] == "TRI"] == ["TRI_PIPE", "TRI_PIPE"]
    _check64(M, b[:1], x)
    x3, _ = _solve(M, b, depth=1)
    _check64(M, b, x3)


@pytest.mark.parametrize("depth", [1, 3])
@pytest.mark.parametrize("dtype", [torch.float64, torch.float32])
@pytest.mark.parametrize("reorder", [False, True])
def test_square_row_blocks(gpu, depth, dtype, reorder):
    """The B200 row-block square kernel on rows of every length class:
    empty, short, 257-1024 entries (one warp alone) and > 1024 entries (split
    into chunks with atomic partial sums)."""
    M = g.shape_long_rows()
    b = g.gen_rhs(M.n, 1)
    x, plan = _solve(M, b, dtype=dtype, depth=depth, reorder=reorder, force_sq_impl="SQ_ADAPT")
    sqs = [s for s in plan.segments() if s["kind"] == "SQ"]
    assert sqs and all(s["impl"] == "SQ_ADAPT" for s in sqs)
    if dtype == torch.float64:
        _check64(M, b, x)
    else:
        assert on.rel_err(x, on.solve(M, b)) <= TOL32


@pytest.mark.parametrize("transpose", [False, True])
@pytest.mark.parametrize("n", [9000, 20000])
def test_row_with_more_than_32_pieces(gpu, n, transpose):
    """A row longer than 32 * kSfNB (8,192) entries is cut into > 32 pieces;
    its last piece adds the partial sums 32 at a time (C3^T has rows of 258K
    entries: the round-2 bug summed only the first 32 pieces)."""
    M = g.shape_arrow(n)
    b = g.gen_rhs(M.n, 1)
    x, plan = _solve(M, b, depth=0, force_tri_impl="TRI_SYNCFREE", transpose=transpose)
    _check64(g.transpose(M) if transpose else M, b, x)


def test_full_size_c2_default_plan(gpu):
    """BASELINE configs[1] at full size with the library defaults: the B200
    depth rules (R30 / R33) keep the 1,999-level root whole and the strand
    wavefront solves it; every component matches the oracle."""
    M, b = g.gen_config("C2", nrhs=1)
    x, plan = _solve(M, b)
    info = plan.info()
    assert info["depth"] == 0 and info["depth_rule"] in (1, 3)
    assert [s["impl"] for s in plan.segments()] == ["TRI_PIPE"]
    _check64(M, b, x)


@pytest.mark.parametrize("cs", [4, 16])
def test_cluster_level_set_experiment(gpu, cs, monkeypatch):
    """DESIGN 5.5: the level-set on one thread-block cluster (k::tri_level_cluster,
    SPTRSV_SF_CLUSTER, not selected by default: measured slower) stays correct,
    including rows cut into pieces within a level."""
    monkeypatch.setenv("SPTRSV_SF_CLUSTER", str(cs))
    M, b = g.gen_config("C3", small=True, nrhs=1)
    x, _ = _solve(M, b, depth=2)
    _check64(M, b, x)
    A = g.shape_arrow(12000)
    bA = g.gen_rhs(A.n, 1)
    x, _ = _solve(A, bA, depth=0, force_tri_impl="TRI_SYNCFREE")
    _check64(A, bA, x)

