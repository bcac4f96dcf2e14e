"""Per-segment times of one config under the two device-memory sources of a
plan (torch caching allocator vs cudaMalloc), same analysis, L2 flushed."""
import os, sys
import numpy as np
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
import paper_conf_icpp_lun020_b200 as sp  # noqa: E402
from workloads import generators as g  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "C5"
nrhs = int(os.environ.get("PROBE_NRHS", "512"))
M = g.gen_matrix(cfg)
b = g.gen_rhs(M.n, nrhs, seed=g.config_seed(cfg))
B = torch.from_numpy(b).cuda().T if nrhs > 1 else torch.from_numpy(b[0]).cuda()
flush = torch.empty(64 << 20, dtype=torch.float32, device="cuda")
for alloc in [None, "torch", None, "torch"]:
    plan = sp.sptrsv_analyse(M.row_ptr, M.col_idx, M.val, graphs=False, allocator=alloc, max_nrhs=nrhs)
    X = torch.empty_like(B)
    for _ in range(2):
        sp.sptrsv_solve(plan, B, X)
    plan.set_profiling(True)
    acc = []
    for _ in range(3):
        flush.zero_()
        sp.sptrsv_solve(plan, B, X)
        acc.append(plan.seg_times())
    plan.set_profiling(False)
    torch.cuda.synchronize()
    t = np.mean(acc, axis=0)
    print(f"alloc={alloc}: total {t.sum():.3f} ms |", " ".join(f"{v:.3f}" for v in t), flush=True)
    plan.free()
    del X
    torch.cuda.empty_cache()
