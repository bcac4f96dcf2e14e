#!/bin/bash
# >32-piece fix (C3^T), transposed timings, pipelined square kernel sweep
O=gpurun_out/r2x
mkdir -p $O
export SPTRSV_GEN_CACHE=/tmp/gencache
timeout 1200 python -m pytest tests/test_gpu_parity.py -q -x -k "more_than_32 or full_size_transpose or square_row_blocks or forced_kernels" > $O/pytest.log 2>&1; echo "pytest rc=$?"; tail -3 $O/pytest.log
timeout 1200 python scripts/time_transposed.py C2 C3 C4 --out $O/transposed.json 2>&1 | tail -3
for pc in 0 2 3 4; do echo "== SQ_PIPE=$pc"; SPTRSV_SQ_PIPE=$pc timeout 600 python scripts/sweep_sf.py C3 2>&1 | tail -1; done
SPTRSV_SQ_PIPE=3 timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "square_row_blocks or (forced_kernels and SQ_ADAPT)" > $O/pytest_pipe.log 2>&1; echo "pytest pipe rc=$?"; tail -2 $O/pytest_pipe.log
