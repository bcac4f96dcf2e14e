"""GPU tests of the device-resident analysis (SURVEY.md 8(f) f-2,
analyse_dev.cu): the plan analysed on the GPU from a device CSR must be the
host analysis's plan bit for bit (plan hash over the permutation, 1/d and
every stored block; segment descriptors, levels, in-degrees, level pointers,
DCSR rows), equal to the structural oracle, and solve to the CPU oracle."""
import numpy as np
import pytest
import torch

import paper_conf_icpp_lun020_b200 as sp
from paper_conf_icpp_lun020_b200 import _capi as C
from oracle import numeric as on
from oracle import structure as st
from workloads import generators as g

pytestmark = pytest.mark.gpu
TOL64, TOL32 = 1e-10, 1e-4


def _dev_csr(M, dtype=np.float64):
    return (torch.from_numpy(M.row_ptr).cuda(), torch.from_numpy(M.col_idx).cuda(),
            torch.from_numpy(M.val.astype(dtype)).cuda())


def _same_plan(a, b):
    assert a.hash() == b.hash()
    assert np.array_equal(a.perm(), b.perm())
    assert np.array_equal(a.levels(), b.levels())
    sa, sb = a.segments(), b.segments()
    assert sa == sb
    for i, s in enumerate(sa):
        if s["kind"] == "TRI":
            for w in (C.ARRAY_IN_DEGREE, C.ARRAY_LEVEL_PTR):
                assert np.array_equal(a.seg_array(i, w), b.seg_array(i, w))
        else:
            assert np.array_equal(a.seg_array(i, C.ARRAY_DCSR_ROWS), b.seg_array(i, C.ARRAY_DCSR_ROWS))


@pytest.mark.parametrize("name", ["C1", "C2", "C3", "C4", "C5"])
@pytest.mark.parametrize("variant", ["REC", "COL", "ROW"])
def test_device_plan_equals_host_plan(gpu, name, variant):
    M, b = g.gen_config(name, small=True, nrhs=1)
    kw = dict(variant=variant, min_block_rows=max(2, M.n // 9))
    ph = sp.sptrsv_analyse(M.row_ptr, M.col_idx, M.val, analysis="host", **kw)
    pd = sp.sptrsv_analyse(*_dev_csr(M), **kw)
    assert ph.info()["analysis"] == 0 and pd.info()["analysis"] in (1, 2)
    _same_plan(ph, pd)
    x = sp.sptrsv_solve(pd, torch.from_numpy(b[0]).cuda())
    torch.cuda.synchronize()
    assert on.rel_err(x.cpu().numpy()[None], on.solve(M, b)) <= TOL64
    ph.free()
    pd.free()


@pytest.mark.parametrize("name", ["C1", "C3", "C5"])
def test_device_plan_matches_structural_oracle(gpu, name):
    M, _ = g.gen_config(name, small=True, nrhs=1)
    pd = sp.sptrsv_analyse(*_dev_csr(M), min_block_rows=max(2, M.n // 9))
    info = pd.info()
    # at these small sizes the narrow-level triangles take the chain kernel,
    # whose stage format is finished on the host (analysis 2); the full-size
    # C3 / C5 plans are device-built end to end (test_full_size_device_analysis)
    assert info["analysis"] in (1, 2)
    A = st.analyse(M, depth=info["depth"], reorder=info["reorder"] == 0)
    assert np.array_equal(pd.perm(), A.perm)
    assert np.array_equal(pd.levels(), A.leaf_level)
    segs = pd.segments()
    assert [(s["row0"], s["row1"], s["col0"], s["col1"], s["nnz"], s["nlevels"], s["kernel"]) for s in segs] == \
        [(o.row0, o.row1, o.col0, o.col1, o.nnz, o.nlevels, o.kernel) for o in A.segs]
    for i, (s, arrs) in enumerate(zip(segs, A.seg_arrays)):
        if s["kind"] == "TRI":
            assert np.array_equal(pd.seg_array(i, C.ARRAY_IN_DEGREE), arrs["IN_DEGREE"])
            assert np.array_equal(pd.seg_array(i, C.ARRAY_LEVEL_PTR), arrs["LEVEL_PTR"])
        else:
            assert np.array_equal(pd.seg_array(i, C.ARRAY_DCSR_ROWS), arrs["DCSR_ROWS"])
    if info["analysis"] == 1:
        with pytest.raises(sp.SptrsvError):
            pd.matrix()  # no host P L P^T for device-built plans
    pd.free()


@pytest.mark.parametrize("name", ["C1", "C3", "C5"])
def test_device_analysis_upper_fp32_multi(gpu, name):
    M, b = g.gen_config(name, small=True, nrhs=3)
    U = g.to_upper(M)
    ph = sp.sptrsv_analyse(U.row_ptr, U.col_idx, U.val, fill="U", analysis="host")
    pd = sp.sptrsv_analyse(*_dev_csr(U), fill="U")
    _same_plan(ph, pd)
    X = sp.sptrsv_solve(pd, torch.from_numpy(b).cuda().T)
    torch.cuda.synchronize()
    assert on.rel_err(X.T.cpu().numpy(), on.solve(U, b)) <= TOL64
    pf = sp.sptrsv_analyse(*_dev_csr(M, np.float32))
    pfh = sp.sptrsv_analyse(M.row_ptr, M.col_idx, M.val.astype(np.float32), analysis="host")
    _same_plan(pf, pfh)
    x = sp.sptrsv_solve(pf, torch.from_numpy(b[0]).float().cuda())
    torch.cuda.synchronize()
    assert on.rel_err(x.double().cpu().numpy()[None], on.solve(M, b[:1])) <= TOL32
    for p in (ph, pd, pf, pfh):
        p.free()


def test_device_analysis_from_host_csr_and_reorder_none(gpu):
    M, b = g.gen_config("C3", small=True, nrhs=1)
    ph = sp.sptrsv_analyse(M.row_ptr, M.col_idx, M.val, analysis="host", reorder=False, depth=2)
    pd = sp.sptrsv_analyse(M.row_ptr, M.col_idx, M.val, analysis="device", reorder=False, depth=2)
    assert pd.info()["analysis"] == 1
    _same_plan(ph, pd)
    ph.free()
    pd.free()


CASES = [
    ("L", [0, 1, 3], [0, 1, 0], [1.0, 1.0, 1.0]),          # row 1 cols 1,0: UNSORTED
    ("L", [0, 1, 3], [0, 0, 0], [1.0, 1.0, 1.0]),          # duplicate: UNSORTED
    ("L", [0, 2, 3], [0, 1, 1], [1.0, 2.0, 1.0]),          # (0,1) above the diagonal
    ("L", [0, 1, 2], [0, 0], [1.0, 2.0]),                  # row 1 has no diagonal
    ("L", [0, 1, 3], [0, 0, 1], [1.0, 2.0, 0.0]),          # zero diagonal
    ("U", [0, 1, 3], [0, 0, 1], [1.0, 2.0, 1.0]),          # (1,0) below the diagonal of U
    ("L", [0, 1, 3], [0, 0, 5], [1.0, 2.0, 1.0]),          # column out of range
    ("L", [1, 1, 3], [0, 0, 1], [1.0, 2.0, 1.0]),          # row_ptr[0] != 0
    ("L", [0, 1, 0, 3], [0, 0, 1], [1.0, 2.0, 1.0]),       # row_ptr not monotone
    ("L", [0, 1, 2, 4], [0, 1, 0, 1], [1.0, 1.0, 1.0, 1.0]),  # row 2: entry above (names the row)
]


@pytest.mark.parametrize("case", range(len(CASES)))
def test_device_validation_matches_host(gpu, case):
    """Same status and the same message (naming the same, lowest bad row) as
    the host analysis."""
    fill, rp, ci, va = CASES[case]
    rp, ci, va = np.array(rp, np.int32), np.array(ci, np.int32), np.array(va)
    errs = []
    for where in ("host", "device"):
        try:
            sp.sptrsv_analyse(rp, ci, va, fill=fill, analysis=where).free()
            errs.append(None)
        except sp.SptrsvError as ex:
            errs.append((ex.status_name, str(ex).split(": ", 2)[-1]))
    assert errs[0] is not None and errs[0] == errs[1], errs


def test_device_validation_lowest_bad_row(gpu):
    M = g.c5_random_multirhs(n=150_001)
    ci, val = M.col_idx.copy(), M.val.copy()
    r_zero, r_unsorted = 120_003, 100_001  # zero pivot late, unsorted earlier
    val[M.row_ptr[r_zero + 1] - 1] = 0.0
    a = M.row_ptr[r_unsorted]
    ci[a], ci[a + 1] = ci[a + 1], ci[a]
    with pytest.raises(sp.SptrsvError) as e:
        sp.sptrsv_analyse(M.row_ptr, ci, val, analysis="device")
    assert e.value.status_name == "UNSORTED" and f"row {r_unsorted}" in str(e.value)


@pytest.mark.parametrize("name", ["C3", "C5", "C2"])
def test_full_size_device_analysis(gpu, name):
    """BASELINE sizes: the device plan is the host plan (hash) and solves to
    the oracle; C2's wavefront formats are finished on the host (analysis 2)."""
    M, b = g.gen_config(name, nrhs=1)
    pd = sp.sptrsv_analyse(*_dev_csr(M))
    ph = sp.sptrsv_analyse(M.row_ptr, M.col_idx, M.val, analysis="host")
    assert pd.hash() == ph.hash()
    assert pd.info()["analysis"] == (2 if name == "C2" else 1)
    x = sp.sptrsv_solve(pd, torch.from_numpy(b[0]).cuda())
    torch.cuda.synchronize()
    assert on.rel_err(x.cpu().numpy()[None], on.solve(M, b)) <= TOL64
    pd.free()
    ph.free()
