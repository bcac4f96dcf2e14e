"""Run a few solves of one config (for ncu / nsys-style captures)."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import argparse
import torch
import paper_conf_icpp_lun020_b200 as sp
from workloads import generators as g

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="C2")
ap.add_argument("--reps", type=int, default=3)
ap.add_argument("--nrhs", type=int, default=None)
ap.add_argument("--selector", default="B200")
ap.add_argument("--force-tri", default=None)
a = ap.parse_args()
M, b = g.gen_config(a.config, nrhs=a.nrhs or 1)
plan = sp.sptrsv_analyse(M.row_ptr, M.col_idx, M.val, selector=a.selector, force_tri_impl=a.force_tri)
B = torch.from_numpy(b).cuda().T
if B.shape[1] == 1:
    B = B[:, 0].contiguous()
flush = torch.empty(64 * 1024 * 1024, dtype=torch.float32, device="cuda")
for _ in range(a.reps):
    flush.zero_()
    X = sp.sptrsv_solve(plan, B)
torch.cuda.synchronize()
print("segments", [(s["kind"], s["impl"], s["nlevels"]) for s in plan.segments()])
