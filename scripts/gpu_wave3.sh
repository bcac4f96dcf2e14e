#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
for d in 0 10; do
mkdir -p gpurun_out/tr$d
SPTRSV_WAVE_DBG=$d SPTRSV_TRACE=1 SPTRSV_TRACE_DIR=gpurun_out/tr$d timeout 300 python scripts/prof_solve.py --config C2 --reps 3 > gpurun_out/trace.log 2>&1; echo "trace rc=$?"
done
