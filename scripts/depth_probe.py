"""Solve time of one config at several recursion depths (PROBE_NRHS right-hand sides) (B200 selector, L2
flushed, CUDA events around whole solves; graphs off).

    python scripts/depth_probe.py C3 0 1 2 3 4
"""
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_icpp_lun020_b200 as sp  # noqa: E402
from oracle import numeric as on  # noqa: E402
from workloads import generators as g  # noqa: E402

cfg = sys.argv[1]
nrhs = int(os.environ.get("PROBE_NRHS", "1"))
M, b = g.gen_config(cfg, nrhs=nrhs)
cols = [0, nrhs - 1]
ref = on.solve(M, b[cols], threads=2)
B = torch.from_numpy(b[0]).cuda() if nrhs == 1 else torch.from_numpy(b).cuda().T
X = torch.empty_like(B)
flush = torch.empty(64 << 20, dtype=torch.float32, device="cuda")
for d in [int(a) for a in sys.argv[2:]]:
    plan = sp.sptrsv_analyse(M.row_ptr, M.col_idx, M.val, depth=d, graphs=False)
    for _ in range(3):
        sp.sptrsv_solve(plan, B, X)
    ts = []
    for _ in range(10):
        flush.zero_()
        e0 = torch.cuda.Event(enable_timing=True)
        e1 = torch.cuda.Event(enable_timing=True)
        e0.record()
        sp.sptrsv_solve(plan, B, X)
        e1.record()
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1))
    xh = X.cpu().numpy()
    err = on.rel_err(xh[None] if nrhs == 1 else xh.T[cols], ref)
    segs = plan.segments()
    print(f"{cfg} nrhs {nrhs} depth {d}: median {np.median(ts):.3f} ms  segs {len(segs)}  "
          f"impls {sorted(set(s['impl'] for s in segs))}  err {err:.1e}", flush=True)
    plan.free()
