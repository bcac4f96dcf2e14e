"""Time sptrsv_analyse (host analysis + upload) of one config, 1 warm-up + 3."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_icpp_lun020_b200 as sp
from workloads import generators as g
c = sys.argv[1]
M = g.gen_matrix(c)
ts = []
for i in range(4):
    t0 = time.perf_counter()
    p = sp.sptrsv_analyse(M.row_ptr, M.col_idx, M.val)
    torch.cuda.synchronize()
    ts.append((time.perf_counter() - t0) * 1e3)
    p.free()
print(c, "analyse ms", [round(t, 1) for t in ts])
