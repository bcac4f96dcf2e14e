"""Per-segment CUDA-event times of repeated solves (tuning helper; no parity)."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import argparse
import numpy as np
import torch
import paper_conf_icpp_lun020_b200 as sp
from workloads import generators as g

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="C2")
ap.add_argument("--reps", type=int, default=20)
ap.add_argument("--nrhs", type=int, default=None)
ap.add_argument("--tag", default="")
ap.add_argument("--depth", type=int, default=-1)
a = ap.parse_args()
M, b = g.gen_config(a.config, nrhs=a.nrhs or 1)
plan = sp.sptrsv_analyse(M.row_ptr, M.col_idx, M.val, depth=a.depth)
B = torch.from_numpy(b).cuda().T
if B.shape[1] == 1:
    B = B[:, 0].contiguous()
flush = torch.empty(64 * 1024 * 1024, dtype=torch.float32, device="cuda")
plan.set_profiling(True)
acc = []
for i in range(a.reps + 3):
    flush.zero_()
    X = sp.sptrsv_solve(plan, B)
    torch.cuda.synchronize()
    if i >= 3:
        acc.append(plan.seg_times())
t = np.mean(acc, axis=0)
names = ["permute_in"] + [f"{s['kind']}:{s['impl']}" for s in plan.segments()] + ["permute_out"]
print(a.tag, "total %.4f ms |" % t.sum(), " ".join(f"{n}={v:.4f}" for n, v in zip(names, t)))
