"""The NCCL path of the multi-RHS sharding (dist.py) on a
B200: dist_solve over a real NCCL process group (world size 1 on the single
GPU the round has; 2 if present) with the CUDA solve, every column checked
against the oracle.  Each case runs in a child process (own process group)."""
import os
import socket
import subprocess
import sys
import textwrap

import pytest
import torch

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _run(world, cfg, nrhs, small):
    code = textwrap.dedent(f"""
        import os, sys
        sys.path.insert(0, {ROOT!r})
        import numpy as np, torch, torch.distributed as dist
        import torch.multiprocessing as mp

        def worker(rank):
            os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT="{_port()}")
            torch.cuda.set_device(rank)
            dist.init_process_group("nccl", rank=rank, world_size={world}, device_id=torch.device("cuda", rank))
            import paper_conf_icpp_lun020_b200 as sp
            from paper_conf_icpp_lun020_b200.dist import check_replicated, dist_solve
            from oracle import numeric as on
            from workloads import generators as g
            M, b = g.gen_config("{cfg}", small={small}, nrhs={nrhs})
            plan = sp.sptrsv_analyse(M.row_ptr, M.col_idx, M.val)
            check_replicated(plan)
            B = torch.from_numpy(b).cuda().T if rank == 0 else None
            X = dist_solve(plan, B, nrhs=None if rank == 0 else {nrhs})
            torch.cuda.synchronize()
            if rank == 0:
                assert X.stride(0) == 1 and X.shape == (M.n, {nrhs})
                xs = X.T.cpu().numpy()
                del X, B
                ref = on.solve(M, b, threads=max(1, len(os.sched_getaffinity(0))))
                errs = [on.rel_err(xs[c], ref[c]) for c in range({nrhs})]
                print("MAXERR", max(errs), "COLS", len(errs), flush=True)
            dist.destroy_process_group()

        if {world} == 1:
            worker(0)
        else:
            mp.spawn(worker, nprocs={world})
    """)
    out = subprocess.run([sys.executable, "-c", code], capture_output=True, text=True, timeout=1200)
    line = [l for l in out.stdout.splitlines() if l.startswith("MAXERR")]
    assert line, out.stdout[-2000:] + out.stderr[-4000:]
    _, err, _, cols = line[0].split()
    return float(err), int(cols)


@pytest.mark.parametrize("nrhs", [37, 1])
def test_dist_solve_nccl_small(gpu, nrhs):
    err, cols = _run(1, "C5", nrhs, True)
    assert cols == nrhs and err <= 1e-10


def test_dist_solve_nccl_full_c5_all_columns(gpu):
    """C5 at full size (n = 2M, 512 RHS) through NCCL scatter / solve /
    gather; all 512 columns against the oracle."""
    err, cols = _run(1, "C5", 512, False)
    assert cols == 512 and err <= 1e-10


@pytest.mark.skipif(torch.cuda.device_count() < 2, reason="needs two GPUs")
def test_dist_solve_nccl_world2_ragged(gpu):
    err, cols = _run(2, "C5", 37, True)
    assert cols == 37 and err <= 1e-10
