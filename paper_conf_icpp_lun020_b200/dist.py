"""Multi-GPU SpTRSM by right-hand-side sharding.

A single triangular solve does not shard: every triangle of Alg 7 (PAPER.md:
L265-L296) depends on the x of the previous segment.  Independent RHS columns
do: rank r of P owns columns [r*k/P, (r+1)*k/P) of B (one contiguous buffer of
a column-major B), solves them with its own replica of the plan, and NCCL
(torch.distributed over NVLink / NVSwitch) is used only to scatter B from the
root and gather X back.  There is no collective inside the solve.

    plan = sp.sptrsv_analyse(...)              # every rank, same CSR
    check_replicated(plan, group)              # all_reduce MIN == MAX of the plan hash
    X = dist_solve(plan, B, group, root=0)     # B / X: (n, k) column-major on the root

Everything numeric happens in the CUDA library (sptrsv_solve); this module
only computes shard bounds and moves buffers.
"""
from __future__ import annotations

from typing import Callable

import torch
import torch.distributed as dist


def shard_bounds(nrhs: int, world: int, rank: int) -> tuple[int, int]:
    """Columns [c0, c1) owned by `rank` (contiguous, sizes differ by <= 1)."""
    if world < 1 or not 0 <= rank < world:
        raise ValueError("bad world/rank")
    return nrhs * rank // world, nrhs * (rank + 1) // world


def check_replicated(plan, group=None) -> int:
    """All ranks must hold the bit-identical plan (deterministic analysis).
    Returns the hash; raises if any rank differs."""
    h = plan.hash()
    # the 64-bit digest travels as two int64 halves (NCCL/gloo reduce signed ints)
    v = torch.tensor([h & 0xFFFFFFFF, h >> 32], dtype=torch.int64)
    if dist.get_backend(group) == "nccl":
        v = v.cuda()
    lo, hi = v.clone(), v.clone()
    dist.all_reduce(lo, op=dist.ReduceOp.MIN, group=group)
    dist.all_reduce(hi, op=dist.ReduceOp.MAX, group=group)
    if not torch.equal(lo, hi):
        raise RuntimeError("replicated plans differ across ranks (analysis not deterministic?)")
    return h


def dist_solve(plan, B: torch.Tensor | None, group=None, root: int = 0, nrhs: int | None = None,
               solve_fn: Callable | None = None) -> torch.Tensor | None:
    """Solve L X = B with the columns of B sharded over the ranks of `group`.

    B: on the root, an (n, k) column-major tensor (B.T contiguous) on the
    rank's device (NCCL) or CPU (gloo); ignored elsewhere (pass None and nrhs=k).
    Returns X (n, k) column-major on the root, None on the other ranks.
    `solve_fn(plan, B_shard) -> X_shard` defaults to the CUDA library's
    sptrsv_solve; the CPU tests substitute a host solver to exercise the
    sharding and the collectives with gloo.
    """
    if solve_fn is None:
        from . import sptrsv_solve as solve_fn  # noqa: N813
    world = dist.get_world_size(group)
    rank = dist.get_rank(group)
    groot = dist.get_global_rank(group, root) if group is not None else root
    n = plan.n
    if rank == root:
        if B.dim() != 2 or B.shape[0] != n or B.stride(0) != 1:
            raise ValueError("B must be (n, k) column-major on the root")
        k = B.shape[1]
        dev, dtype = B.device, B.dtype
        meta = torch.tensor([k, 0 if dtype == torch.float64 else 1], dtype=torch.int64)
    else:
        meta = torch.zeros(2, dtype=torch.int64)
    nccl = dist.get_backend(group) == "nccl"
    if nccl:
        meta = meta.cuda()
    dist.broadcast(meta, src=groot, group=group)
    k = int(meta[0].item())
    dtype = torch.float64 if int(meta[1].item()) == 0 else torch.float32
    dev = torch.device("cuda", torch.cuda.current_device()) if nccl else torch.device("cpu")
    if nrhs is not None and nrhs != k:
        raise ValueError(f"nrhs={nrhs} but the root's B has {k} columns")
    c0, c1 = shard_bounds(k, world, rank)
    even = k % world == 0 and (rank != root or B.stride(1) == n)  # root: B.T rows contiguous
    # equal-size shards for scatter/gather: when P divides k the column-major
    # shards are contiguous row blocks of B.T / X.T and travel as views (no
    # staging copy); otherwise every shard is padded to ceil(k / P) columns
    w = -(-k // world)
    mine = torch.empty(w, n, dtype=dtype, device=dev)  # row c = column c of the shard
    scatter_list = None
    if rank == root:
        bt = B.T  # (k, n) row-major view: column c of B is row c, contiguous
        scatter_list = []
        for r in range(world):
            a, b = shard_bounds(k, world, r)
            if even:
                scatter_list.append(bt[a:b])
            else:
                buf = torch.zeros(w, n, dtype=dtype, device=dev)
                buf[: b - a].copy_(bt[a:b])
                scatter_list.append(buf)
    dist.scatter(mine, scatter_list, src=groot, group=group)
    xs = torch.empty_like(mine)
    if c1 > c0:
        b_shard = mine[: c1 - c0].T  # (n, c1-c0) column-major
        x_out = xs[: c1 - c0].T
        if c1 - c0 == 1:
            b_shard, x_out = b_shard[:, 0], x_out[:, 0]
        x_shard = solve_fn(plan, b_shard, x_out) if _takes_out(solve_fn) else solve_fn(plan, b_shard)
        if x_shard is not None and x_shard.data_ptr() != x_out.data_ptr():
            x_out.copy_(x_shard)
    X = torch.empty(k, n, dtype=dtype, device=dev) if rank == root else None
    if rank == root and even:
        gather_list = [X[a:b] for a, b in (shard_bounds(k, world, r) for r in range(world))]
    else:
        gather_list = [torch.empty_like(mine) for _ in range(world)] if rank == root else None
    dist.gather(xs, gather_list, dst=groot, group=group)
    if rank != root:
        return None
    if not even:
        for r in range(world):
            a, b = shard_bounds(k, world, r)
            X[a:b].copy_(gather_list[r][: b - a])
    return X.T


def _takes_out(fn) -> bool:
    """solve_fn(plan, b, x) writes into x (the CUDA library's sptrsv_solve)."""
    try:
        import inspect
        return len(inspect.signature(fn).parameters) >= 3
    except (TypeError, ValueError):
        return False
