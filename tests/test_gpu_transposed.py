"""A^T x = b from the SAME plan (R32; C ABI
sptrsv_solve_transposed): the push-form sync-free solve (Alg 3, PAPER.md
L105-L125, atomics on left_sum and in-degree) over the plan's segments in
reverse order, against the oracle's substitution on the explicitly
transposed matrix (g.transpose -> oracle Alg 1 / backward substitution)."""
import numpy as np
import pytest
import torch

import paper_conf_icpp_lun020_b200 as sp
from oracle import numeric as on
from workloads import generators as g

pytestmark = pytest.mark.gpu
TOL64, TOL32 = 1e-10, 1e-4


def _solve_T(M, b1, dtype=torch.float64, **kw):
    """b1: numpy (n,).  Returns (x numpy float64 (n,), plan)."""
    val = M.val if dtype == torch.float64 else M.val.astype(np.float32)
    plan = sp.sptrsv_analyse(M.row_ptr, M.col_idx, val, fill=M.uplo, **kw)
    B = torch.from_numpy(b1).to("cuda", dtype)
    X = sp.sptrsv_solve(plan, B, transposed=True)
    torch.cuda.synchronize()
    return X.double().cpu().numpy(), plan


def _check(M, b1, x, tol=TOL64):
    MT = g.transpose(M)
    ref = on.solve(MT, b1[None])
    err = on.rel_err(x[None], ref)
    assert err <= tol, err
    if tol == TOL64:
        ok, worst = on.residual_bound_ok(MT, x[None], b1[None])
        assert ok, worst


CONFIGS = ["C1", "C2", "C3", "C4", "C5"]


@pytest.mark.parametrize("name", CONFIGS)
@pytest.mark.parametrize("uplo", ["L", "U"])
@pytest.mark.parametrize("variant", ["REC", "COL", "ROW"])
def test_transposed_same_plan(gpu, name, uplo, variant):
    M, b = g.gen_config(name, small=True, nrhs=1)
    if uplo == "U":
        M = g.to_upper(M)
    x, _ = _solve_T(M, b[0], depth=2, variant=variant)
    _check(M, b[0], x)


@pytest.mark.parametrize("name", CONFIGS)
@pytest.mark.parametrize("tri", ["TRI_LEVELSET", "TRI_SYNCFREE", "TRI_CHAIN", "TRI_SUPERNODE", "TRI_PIPE"])
def test_transposed_every_forward_format(gpu, name, tri):
    """The transposed sweep reads the CSR every triangle format keeps -- also
    the wave triangles' strand-ordered device rows (claim order array)."""
    M, b = g.gen_config(name, small=True, nrhs=1)
    x, plan = _solve_T(M, b[0], depth=2, force_tri_impl=tri)
    _check(M, b[0], x)


@pytest.mark.parametrize("name", ["C1", "C3", "C5"])
def test_transposed_fp32_and_paper_selector(gpu, name):
    M, b = g.gen_config(name, small=True, nrhs=1)
    x, _ = _solve_T(M, b[0], dtype=torch.float32, depth=3)
    _check(M, b[0], x, TOL32)
    x, _ = _solve_T(M, b[0], selector="PAPER", depth=1)
    _check(M, b[0], x)


def test_transposed_repeat_inplace_and_forward_interleaved(gpu):
    """Counters and tickets are reset by every solve; forward and transposed
    solves share the plan's workspace; b == x in place."""
    M, b = g.gen_config("C3", small=True, nrhs=1)
    plan = sp.sptrsv_analyse(M.row_ptr, M.col_idx, M.val, depth=3)
    B = torch.from_numpy(b[0]).cuda()
    ref_t = on.solve(g.transpose(M), b)
    ref_f = on.solve(M, b)
    for _ in range(3):
        xt = sp.sptrsv_solve(plan, B, transposed=True)
        xf = sp.sptrsv_solve(plan, B)
        torch.cuda.synchronize()
        assert on.rel_err(xt.cpu().numpy()[None], ref_t) <= TOL64
        assert on.rel_err(xf.cpu().numpy()[None], ref_f) <= TOL64
    Bi = B.clone()
    sp.sptrsv_solve(plan, Bi, Bi, transposed=True)
    torch.cuda.synchronize()
    assert on.rel_err(Bi.cpu().numpy()[None], ref_t) <= TOL64


def test_transposed_of_transposed_plan_is_forward(gpu):
    """A plan analysed with transpose=1 solves A^T x = b; its transposed solve
    is A x = b again."""
    M, b = g.gen_config("C1", small=True, nrhs=1)
    plan = sp.sptrsv_analyse(M.row_ptr, M.col_idx, M.val, transpose=True)
    x = sp.sptrsv_solve(plan, torch.from_numpy(b[0]).cuda(), transposed=True)
    torch.cuda.synchronize()
    assert on.rel_err(x.cpu().numpy()[None], on.solve(M, b)) <= TOL64


def test_transposed_errors(gpu):
    M, b = g.gen_config("C1", small=True, nrhs=2)
    plan = sp.sptrsv_analyse(M.row_ptr, M.col_idx, M.val)
    with pytest.raises(RuntimeError, match="NOT_SUPPORTED"):
        sp.sptrsv_solve(plan, torch.from_numpy(b).cuda().T, transposed=True)  # two RHS
    with pytest.raises(RuntimeError, match="NOT_SUPPORTED"):
        sp.sptrsv_solve(plan, b[0].copy(), transposed=True)  # host pointers


@pytest.mark.parametrize("name", ["C2", "C3", "C4", "C5"])
def test_full_size_transposed_same_plan(gpu, name):
    """Full BASELINE sizes, default options."""
    M, b = g.gen_config(name, nrhs=1)
    x, _ = _solve_T(M, b[0])
    MT = g.transpose(M)
    assert on.rel_err(x[None], on.solve(MT, b)) <= TOL64


@pytest.mark.parametrize("name", ["C1", "C2", "C3"])
@pytest.mark.parametrize("chain", [True, False])
def test_transposed_narrow_level_chain(gpu, name, chain, monkeypatch):
    """Narrow-level triangles (every level <= 2,048 rows, >= 32 levels) take
    the one-CTA reverse chain with the shared-memory ring (k::tri_pushchain_T);
    SPTRSV_NO_PUSHCHAIN forces the multi-CTA counter kernel.  Both against
    the oracle, with the wavefront's strand-ordered device rows (C2) and a
    deep bidiagonal chain whose every level is one row."""
    if not chain:
        monkeypatch.setenv("SPTRSV_NO_PUSHCHAIN", "1")
    M, b = g.gen_config(name, small=True, nrhs=1)
    x, _ = _solve_T(M, b[0], depth=1)
    _check(M, b[0], x)
    Mb = g.shape_bidiagonal(3000)
    bb = g.gen_rhs(Mb.n, 1)
    x, _ = _solve_T(Mb, bb[0])
    _check(Mb, bb[0], x)
