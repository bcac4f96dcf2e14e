"""IC(0)-preconditioned conjugate gradients on the C2 workload (SURVEY.md
8(f) f-4): the iterative scenario the paper names as SpTRSV's main use
("preconditioners ... in iterative solvers"; L358-L363 on
amortising the preprocessing over many solves).

A is the 2D 5-point Laplacian (diagonal 4, neighbours -1) and L its exact
IC(0) factor (workloads.generators.c2_laplacian_ic0).  Each CG iteration
applies M^-1 r = L^-T (L^-1 r) with two sptrsv_solve calls: the plan of L and
the plan of L analysed with transpose=True (R31), both preprocessed
once.  This is a DRIVER around the library, not part of its hot path: the
CG vector updates and the A p product are plain torch ops.

  python examples/ic0_pcg.py [--nx 1000] [--tol 1e-8]
"""
from __future__ import annotations

import argparse
import os
import sys
import time

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_icpp_lun020_b200 as sp  # noqa: E402
from workloads import generators as g  # noqa: E402


def laplacian_csr(nx: int, ny: int, device) -> torch.Tensor:
    """The 5-point Laplacian A = L L^T + R (R: IC(0)'s dropped fill) as torch CSR."""
    n = nx * ny
    i = np.arange(n)
    ix, iy = i % nx, i // nx
    rows, cols, vals = [i], [i], [np.full(n, 4.0)]
    for m, off in ((ix > 0, -1), (ix < nx - 1, 1), (iy > 0, -nx), (iy < ny - 1, nx)):
        rows.append(i[m])
        cols.append(i[m] + off)
        vals.append(np.full(int(m.sum()), -1.0))
    r, c, v = (np.concatenate(a) for a in (rows, cols, vals))
    o = np.lexsort((c, r))
    rp = np.zeros(n + 1, dtype=np.int64)
    np.cumsum(np.bincount(r, minlength=n), out=rp[1:])
    return torch.sparse_csr_tensor(torch.from_numpy(rp), torch.from_numpy(c[o]), torch.from_numpy(v[o]),
                                   size=(n, n)).to(device)


class IC0:
    """M^-1 = L^-T L^-1.  same_plan=False (default): two plans analysed once
    (forward, and the analysed transpose, R31: the fast pull-form kernels for
    both sweeps).  same_plan=True: ONE plan; the L^-T sweep is the same
    plan's push-form transposed solve (R32: no second analysis or copy)."""

    def __init__(self, L, same_plan: bool = False):
        self.fwd = sp.sptrsv_analyse(L.row_ptr, L.col_idx, L.val)
        self.same = same_plan
        self.bwd = None if same_plan else sp.sptrsv_analyse(L.row_ptr, L.col_idx, L.val, transpose=True)

    def __call__(self, r: torch.Tensor) -> torch.Tensor:
        y = sp.sptrsv_solve(self.fwd, r)
        if self.same:
            return sp.sptrsv_solve(self.fwd, y, transposed=True)
        return sp.sptrsv_solve(self.bwd, y)

    def free(self):
        self.fwd.free()
        if self.bwd is not None:
            self.bwd.free()


def pcg(A: torch.Tensor, b: torch.Tensor, M=None, tol: float = 1e-8, maxiter: int = 10000):
    """Textbook (P)CG; returns (x, iterations, relative residual history)."""
    x = torch.zeros_like(b)
    r = b.clone()
    z = M(r) if M else r
    p = z.clone()
    rz = torch.dot(r, z)
    nb = torch.linalg.vector_norm(b)
    hist = []
    for it in range(1, maxiter + 1):
        Ap = torch.mv(A, p)
        alpha = rz / torch.dot(p, Ap)
        x += alpha * p
        r -= alpha * Ap
        rel = float(torch.linalg.vector_norm(r) / nb)
        hist.append(rel)
        if rel <= tol:
            return x, it, hist
        z = M(r) if M else r
        rz_new = torch.dot(r, z)
        p = z + (rz_new / rz) * p
        rz = rz_new
    return x, maxiter, hist


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--nx", type=int, default=1000)
    ap.add_argument("--tol", type=float, default=1e-8)
    a = ap.parse_args()
    dev = torch.device("cuda:0")
    L = g.c2_laplacian_ic0(a.nx)
    A = laplacian_csr(a.nx, a.nx, dev)
    b = torch.from_numpy(g.gen_rhs(L.n, 1)[0]).to(dev)
    t0 = time.perf_counter()
    M = IC0(L)
    pre = time.perf_counter() - t0
    for name, prec in (("CG", None), ("IC(0)-PCG", M)):
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        x, it, hist = pcg(A, b, prec, a.tol)
        torch.cuda.synchronize()
        dt = time.perf_counter() - t0
        print(f"{name:10s} n={L.n} iterations={it} rel_res={hist[-1]:.2e} time={dt * 1e3:.1f} ms "
              f"({dt / it * 1e3:.3f} ms/iter)")
    # the two triangular solves of one preconditioner application, device-timed
    r = torch.randn(L.n, dtype=torch.float64, device=dev)
    for _ in range(3):
        M(r)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(20):
        M(r)
    e1.record()
    torch.cuda.synchronize()
    print(f"preconditioner apply (L then L^T solve): {e0.elapsed_time(e1) / 20:.3f} ms; "
          f"preprocessing of both plans {pre * 1e3:.0f} ms")
    M.free()


if __name__ == "__main__":
    main()
