#!/bin/bash
# same-plan transposed solve with the one-CTA reverse chain for narrow levels
O=gpurun_out/r2pc
mkdir -p $O
export SPTRSV_GEN_CACHE=/tmp/gencache
timeout 1200 python -m pytest tests/test_gpu_transposed.py -q -x > $O/pytest_T.log 2>&1; echo "pytest T rc=$?"; tail -2 $O/pytest_T.log
timeout 1200 python scripts/time_transposed.py C2 C3 C4 --out $O/transposed.json 2>&1 | tail -3
python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
