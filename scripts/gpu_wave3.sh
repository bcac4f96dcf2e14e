#!/bin/bash
mkdir -p gpurun_out/tr
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
SPTRSV_TRACE=1 SPTRSV_TRACE_DIR=gpurun_out/tr timeout 300 python scripts/prof_solve.py --config C2 --reps 3 > gpurun_out/trace.log 2>&1; echo "trace rc=$?"
