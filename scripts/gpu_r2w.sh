#!/bin/bash
# transposed push kernels v2 (warp-cooperative long rows, acq_rel fences); Fig. 5 re-derivation evidence
O=gpurun_out/r2w
mkdir -p $O
export SPTRSV_GEN_CACHE=/tmp/gencache
timeout 1200 python -m pytest tests/test_gpu_transposed.py -q -x > $O/pytest_T.log 2>&1; echo "pytest T rc=$?"; tail -3 $O/pytest_T.log
timeout 1200 python scripts/time_transposed.py C2 C3 C4 --out $O/transposed.json 2>&1 | tail -3
timeout 1800 python scripts/fig5_derive.py --quick > $O/fig5.log 2>&1; echo "fig5 rc=$?"; tail -30 $O/fig5.log
cp profiles/r02_fig5.json $O/ 2>/dev/null
