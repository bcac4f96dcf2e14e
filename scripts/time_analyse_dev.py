"""Time sptrsv_analyse with the CSR on the device (f-2) and on the host:
1 warm-up + 3 timed each, with a hash check that both give the same plan."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import paper_conf_icpp_lun020_b200 as sp
from workloads import generators as g
for c in sys.argv[1:]:
    M = g.gen_matrix(c)
    d = [torch.from_numpy(a).cuda() for a in (M.row_ptr, M.col_idx, M.val)]
    torch.cuda.synchronize()
    res = {}
    for where, args in (("device", d), ("host", (M.row_ptr, M.col_idx, M.val))):
        ts = []
        for i in range(4):
            t0 = time.perf_counter()
            p = sp.sptrsv_analyse(*args)
            torch.cuda.synchronize()
            ts.append((time.perf_counter() - t0) * 1e3)
            if i < 3:
                p.free()
        res[where] = (p, ts)
    hd, hh = res["device"][0].hash(), res["host"][0].hash()
    print(c, "device ms", [round(t, 1) for t in res["device"][1]], "analysis", res["device"][0].info()["analysis"],
          "| host ms", [round(t, 1) for t in res["host"][1]], "| same plan", hd == hh, flush=True)
