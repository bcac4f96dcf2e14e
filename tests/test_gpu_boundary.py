"""GPU tests of the C-ABI contract (include/sptrsv.h):
device memory through torch's caching allocator, CUDA-graph replay of
repeated solves, argument checks, the spin-wait watchdog and the
stream-scoped free.  Values are checked against the CPU oracle (Alg 1)."""
import os
import subprocess
import sys
import textwrap

import numpy as np
import pytest
import torch

import paper_conf_icpp_lun020_b200 as sp
from oracle import numeric as on
from workloads import generators as g

pytestmark = pytest.mark.gpu
TOL64 = 1e-10
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_plan_and_workspace_are_torch_memory(gpu):
    """dev_alloc hooks: the arena and the solve workspace are allocated by
    torch's caching allocator (torch.cuda.memory_allocated sees them) and
    returned to it by sptrsv_free."""
    M, b = g.gen_config("C3", small=True, nrhs=4)
    torch.cuda.synchronize()
    m0 = torch.cuda.memory_allocated()
    plan = sp.sptrsv_analyse(M.row_ptr, M.col_idx, M.val, max_nrhs=4)
    info = plan.info()
    m1 = torch.cuda.memory_allocated()
    ws = 2 * M.n * 4 * 8  # bw + xs for 4 RHS
    assert m1 - m0 >= info["device_bytes"] + ws, (m1 - m0, info["device_bytes"], ws)
    B = torch.from_numpy(b).cuda().T
    X = sp.sptrsv_solve(plan, B)
    torch.cuda.synchronize()
    assert on.rel_err(X.T.cpu().numpy(), on.solve(M, b)) <= TOL64
    del X
    m2 = torch.cuda.memory_allocated()
    plan.free()
    m3 = torch.cuda.memory_allocated()
    assert m2 - m3 >= info["device_bytes"] + ws


def test_cudamalloc_allocator_still_works(gpu):
    M, b = g.gen_config("C1", nrhs=2)
    plan = sp.sptrsv_analyse(M.row_ptr, M.col_idx, M.val, allocator=None)
    X = sp.sptrsv_solve(plan, torch.from_numpy(b).cuda().T)
    torch.cuda.synchronize()
    assert on.rel_err(X.T.cpu().numpy(), on.solve(M, b)) <= TOL64
    plan.free()


@pytest.mark.parametrize("name,nrhs", [("C1", 1), ("C2", 1), ("C3", 1), ("C4", 1), ("C5", 5), ("C4", 20)])
def test_graph_replay_matches_oracle(gpu, name, nrhs):
    """A repeated solve with the same buffers is captured (2nd call) and
    replayed (3rd call on): every replay reads the CURRENT b (new values each
    time) and, for multi-RHS, takes a fresh epoch from the device counter."""
    M, _ = g.gen_config(name, small=True, nrhs=1)
    plan = sp.sptrsv_analyse(M.row_ptr, M.col_idx, M.val, min_block_rows=max(2, M.n // 9))
    B = torch.empty((nrhs, M.n), dtype=torch.float64, device="cuda").T  # column-major
    if nrhs == 1:
        B = torch.empty(M.n, dtype=torch.float64, device="cuda")
    X = torch.empty_like(B)
    for it in range(6):
        b = g.gen_rhs(M.n, nrhs, seed=1234 + it)
        bt = torch.from_numpy(b).cuda()  # (nrhs, n)
        B.copy_(bt[0] if nrhs == 1 else bt.T)
        sp.sptrsv_solve(plan, B, X)
        torch.cuda.synchronize()
        x = X.cpu().numpy()
        x = x[None] if nrhs == 1 else x.T
        assert on.rel_err(x, on.solve(M, b)) <= TOL64, it
    plan.free()


def test_graphs_off_and_profiling_agree(gpu):
    M, b = g.gen_config("C3", small=True, nrhs=1)
    outs = []
    for graphs in (True, False):
        plan = sp.sptrsv_analyse(M.row_ptr, M.col_idx, M.val, graphs=graphs)
        B = torch.from_numpy(b[0]).cuda()
        X = torch.empty_like(B)
        for _ in range(3):
            sp.sptrsv_solve(plan, B, X)
        plan.set_profiling(True)
        sp.sptrsv_solve(plan, B, X)
        t = plan.seg_times()
        assert len(t) == len(plan.segments()) + 2 and np.all(t >= 0)
        torch.cuda.synchronize()
        outs.append(X.cpu().numpy())
        plan.free()
    ref = on.solve(M, b)
    for x in outs:
        assert on.rel_err(x[None], ref) <= TOL64


def test_solve_inside_callers_graph_capture(gpu):
    """sptrsv_solve on a stream the caller is capturing enqueues into that
    capture (no nested capture); the caller's graph replays the solve."""
    M, b = g.gen_config("C1", nrhs=1)
    plan = sp.sptrsv_analyse(M.row_ptr, M.col_idx, M.val, max_nrhs=1)
    B = torch.from_numpy(b[0]).cuda()
    X = torch.empty_like(B)
    sp.sptrsv_solve(plan, B, X)  # warm (attributes, workspace)
    torch.cuda.synchronize()
    s = torch.cuda.Stream()
    gr = torch.cuda.CUDAGraph()
    X.zero_()
    with torch.cuda.graph(gr, stream=s):
        sp.sptrsv_solve(plan, B, X, stream=s)
    gr.replay()
    torch.cuda.synchronize()
    assert on.rel_err(X.cpu().numpy()[None], on.solve(M, b)) <= TOL64
    plan.free()


def test_dtype_mismatch_rejected(gpu):
    M, b = g.gen_config("C1", nrhs=1)
    plan = sp.sptrsv_analyse(M.row_ptr, M.col_idx, M.val)
    B = torch.from_numpy(b[0]).cuda()
    with pytest.raises(TypeError):
        sp.sptrsv_solve(plan, B.float())
    with pytest.raises(TypeError):
        sp.sptrsv_solve(plan, B, torch.empty(M.n, dtype=torch.float32, device="cuda"))
    plan.free()


@pytest.mark.skipif(torch.cuda.device_count() < 2, reason="needs two GPUs")
def test_device_mismatch_rejected(gpu):
    M, b = g.gen_config("C1", nrhs=1)
    plan = sp.sptrsv_analyse(M.row_ptr, M.col_idx, M.val, device=0)
    B = torch.from_numpy(b[0]).to("cuda:1")
    with pytest.raises(ValueError):
        sp.sptrsv_solve(plan, B)
    plan.free()


def test_watchdog_reports_deadlock(gpu):
    """SPTRSV_TEST_WEDGE makes one sync-free row depend on itself; the
    spin-wait watchdog (SPTRSV_WATCHDOG_SPINS polls) trips instead of hanging,
    the other warps give up as soon as they see the device copy of the trip,
    and the NEXT call on the plan returns SPTRSV_ERROR_DEADLOCK.  Run in a
    child process: the hooks are read at analysis."""
    code = textwrap.dedent(f"""
        import sys, time; sys.path.insert(0, {ROOT!r})
        import torch, paper_conf_icpp_lun020_b200 as sp
        from workloads import generators as g
        M, b = g.gen_config("C3", small=True, nrhs=1)
        plan = sp.sptrsv_analyse(M.row_ptr, M.col_idx, M.val, force_tri_impl="TRI_SYNCFREE", graphs=False)
        B = torch.from_numpy(b[0]).cuda()
        t0 = time.time()
        sp.sptrsv_solve(plan, B)
        torch.cuda.synchronize()
        dt = time.time() - t0
        try:
            sp.sptrsv_solve(plan, B)
            print("NO_ERROR")
        except sp.SptrsvError as e:
            print("STATUS", e.status_name, round(dt, 2))
        plan.free()
    """)
    env = dict(os.environ, SPTRSV_TEST_WEDGE="1", SPTRSV_WATCHDOG_SPINS="20000")
    out = subprocess.run([sys.executable, "-c", code], env=env, capture_output=True, text=True, timeout=300)
    assert "STATUS DEADLOCK" in out.stdout, out.stdout + out.stderr


def test_free_waits_for_its_stream_only(gpu):
    """sptrsv_free waits on the event recorded after the plan's last solve:
    freeing right after an asynchronous solve on a side stream is safe and
    the result (consumed after the free) is correct."""
    M, b = g.gen_config("C3", small=True, nrhs=1)
    plan = sp.sptrsv_analyse(M.row_ptr, M.col_idx, M.val)
    s = torch.cuda.Stream()
    B = torch.from_numpy(b[0]).cuda()
    torch.cuda.synchronize()
    with torch.cuda.stream(s):
        X = sp.sptrsv_solve(plan, B, stream=s)
    plan.free()
    s.synchronize()
    assert on.rel_err(X.cpu().numpy()[None], on.solve(M, b)) <= TOL64
