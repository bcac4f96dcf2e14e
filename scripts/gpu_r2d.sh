#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
export SPTRSV_GEN_CACHE=/tmp/gencache
echo "== V1"
timeout 900 python scripts/sweep_sf.py C3 SPTRSV_SF_CTAS=16 SPTRSV_SF_CTAS=37 SPTRSV_SF_CTAS=74 SPTRSV_SF_CTAS=148 SPTRSV_SF_CTAS=592 SPTRSV_SF_BACKOFF=0 SPTRSV_SF_BACKOFF=0,SPTRSV_SF_CTAS=37 SPTRSV_SF_BACKOFF=0,SPTRSV_SF_CTAS=74 SPTRSV_SF_BACKOFF=512 SPTRSV_SF_BACKOFF=2000 2>&1 | tail -12
echo "== ITEMS"
SPTRSV_SF_ITEMS=1 timeout 900 python scripts/sweep_sf.py C3 SPTRSV_SF_CTAS=16 SPTRSV_SF_CTAS=37 SPTRSV_SF_CTAS=74 SPTRSV_SF_CTAS=148 SPTRSV_SF_BACKOFF=0 SPTRSV_SF_BACKOFF=0,SPTRSV_SF_CTAS=37 SPTRSV_SF_BACKOFF=512 2>&1 | tail -9
echo "== analyse trace"
for c in C2 C3 C4 C5; do SPTRSV_ANALYSE_TRACE=1 python -c "
import sys,time; sys.path.insert(0,'.')
import torch, paper_conf_icpp_lun020_b200 as sp
from workloads import generators as g
M=g.gen_matrix('$c')
p=sp.sptrsv_analyse(M.row_ptr,M.col_idx,M.val); p.free()
t0=time.perf_counter(); p=sp.sptrsv_analyse(M.row_ptr,M.col_idx,M.val); torch.cuda.synchronize(); print('$c total ms', (time.perf_counter()-t0)*1e3)
" 2>&1 | tail -22; done
