"""Isolated per-group cost of the strand wavefront kernel (tuning helper).

A narrow grid (nx x ny 5-point IC(0) factor, nx <= 32) has <= nx rows per
level, so a single strand (SPTRSV_WAVE=1,1,GPC,NCH) walks one group per
level; ns per level = the kernel's loop time per group with no imports.
Wider clusters (C > 1) add the cross-strand pacing."""
import sys, os, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import argparse
import numpy as np
import torch
import paper_conf_icpp_lun020_b200 as sp
from workloads import generators as g

ap = argparse.ArgumentParser()
ap.add_argument("--nx", type=int, default=32)
ap.add_argument("--ny", type=int, default=20000)
ap.add_argument("--reps", type=int, default=10)
ap.add_argument("--tag", default="")
a = ap.parse_args()
M = g.c2_laplacian_ic0(a.nx, a.ny)
b = g.gen_rhs(M.n, 1)
plan = sp.sptrsv_analyse(M.row_ptr, M.col_idx, M.val, depth=0, force_tri_impl="TRI_PIPE")
segs = plan.segments()
B = torch.from_numpy(b[0]).cuda().contiguous()
plan.set_profiling(True)
ts = []
for i in range(a.reps + 2):
    X = sp.sptrsv_solve(plan, B)
    torch.cuda.synchronize()
    if i >= 2:
        ts.append(plan.seg_times()[1])
t = float(np.median(ts))
nl = segs[0]["nlevels"]
print(f"{a.tag} nx={a.nx} ny={a.ny} impl={segs[0]['impl']} levels={nl} tri={t:.4f} ms  {t * 1e6 / nl:.1f} ns/level "
      f"({t * 1e6 / nl * 1.965:.0f} cycles)")
