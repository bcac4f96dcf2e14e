"""Multi-rank RHS sharding on CPU with gloo, world size 2.

The CUDA solve is replaced by the oracle (tests may call it) so that the
sharding, padding, scatter/gather and plan-hash replication check of
paper_conf_icpp_lun020_b200.dist run without a GPU.  The GPU path of the same
function is exercised by bench.py --config C5 --gpus N (NCCL).
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_icpp_lun020_b200.dist import shard_bounds


def test_shard_bounds_cover_and_balance():
    for k in [0, 1, 5, 64, 512, 513]:
        for P in [1, 2, 3, 8]:
            cols = []
            sizes = []
            for r in range(P):
                a, b = shard_bounds(k, P, r)
                cols.extend(range(a, b))
                sizes.append(b - a)
            assert cols == list(range(k))
            assert max(sizes) - min(sizes) <= 1


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, nrhs, out_q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import paper_conf_icpp_lun020_b200 as sp
        from paper_conf_icpp_lun020_b200.dist import check_replicated, dist_solve
        from oracle import numeric as on
        from workloads import generators as g

        M, b = g.gen_config("C5", small=True, nrhs=nrhs)
        # the analysis runs on the host (no GPU here); every rank builds its own replica
        plan = sp.sptrsv_analyse(M.row_ptr, M.col_idx, M.val, host_only=True, min_block_rows=M.n // 4)
        h = check_replicated(plan)

        def host_solve(plan_, bsh):  # oracle in place of the CUDA solve
            bn = bsh.numpy()
            bn = bn[None] if bn.ndim == 1 else bn.T
            x = on.solve(M, np.ascontiguousarray(bn))
            x = torch.from_numpy(x)
            return x[0] if bsh.dim() == 1 else x.T

        B = torch.from_numpy(b).T if rank == 0 else None  # (n, k) column-major
        X = dist_solve(plan, B, nrhs=None if rank == 0 else nrhs, solve_fn=host_solve)
        if rank == 0:
            ref = on.solve(M, b)
            out_q.put(("ok", float(np.abs(X.T.numpy() - ref).max()), tuple(X.stride()), h))
        else:
            out_q.put(("ok", X is None, None, h))
    except Exception as e:  # pragma: no cover - reported to the parent
        out_q.put(("err", repr(e), None, None))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("nrhs", [5, 1])
def test_dist_solve_gloo_world2(nrhs):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, nrhs, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = [q.get(timeout=300) for _ in range(2)]
    for p in procs:
        p.join(timeout=60)
    assert all(r[0] == "ok" for r in res), res
    root = [r for r in res if r[2] is not None][0]
    other = [r for r in res if r[2] is None][0]
    assert root[1] == 0.0  # the gathered X is exactly the per-column solve
    assert root[2][0] == 1  # column-major (n, k)
    assert other[1] is True  # non-root ranks get None
    assert root[3] == other[3]  # identical plan hash on both ranks
