#!/bin/bash
# transposed solve from the same plan; sq_adapt_1 with hoisted loads
O=gpurun_out/r2v
mkdir -p $O
export SPTRSV_GEN_CACHE=/tmp/gencache
timeout 1200 python -m pytest tests/test_gpu_transposed.py -q -x > $O/pytest_T.log 2>&1; echo "pytest T rc=$?"; tail -15 $O/pytest_T.log | grep -v "^$" | tail -8
timeout 600 python scripts/sweep_sf.py C3 2>&1 | tail -1
timeout 600 python scripts/sweep_sf.py C3 2>&1 | tail -1
python - <<'PY'
import sys, os, time, torch
sys.path.insert(0, os.getcwd())
import paper_conf_icpp_lun020_b200 as sp
from workloads import generators as g
for cfg in ["C2", "C3", "C4"]:
    M, b = g.gen_config(cfg, nrhs=1)
    plan = sp.sptrsv_analyse(M.row_ptr, M.col_idx, M.val)
    B = torch.from_numpy(b[0]).cuda(); X = torch.empty_like(B)
    fl = torch.empty(64 << 20, dtype=torch.float32, device="cuda")
    for _ in range(3): sp.sptrsv_solve(plan, B, X, transposed=True)
    ts = []
    for _ in range(10):
        fl.zero_(); e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
        e0.record(); sp.sptrsv_solve(plan, B, X, transposed=True); e1.record(); torch.cuda.synchronize(); ts.append(e0.elapsed_time(e1))
    ts.sort(); print(cfg, "transposed same plan: median %.3f ms" % ts[len(ts)//2], flush=True)
    plan.free()
PY
