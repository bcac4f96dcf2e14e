#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
timeout 300 python scripts/time_segs.py --config C2 --tag "default" 2>&1 | tail -1
for geo in "8,4,8,4" "16,2,8,4" "16,4,8,3" "16,8,8,4"; do
  SPTRSV_WAVE=$geo timeout 300 python scripts/time_segs.py --config C2 --tag "geo=$geo" 2>&1 | tail -1
done
mkdir -p gpurun_out/tr
SPTRSV_TRACE=1 SPTRSV_TRACE_DIR=gpurun_out/tr timeout 300 python scripts/prof_solve.py --config C2 --reps 3 > gpurun_out/trace.log 2>&1; echo "trace rc=$?"
timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "wave or forced_kernels or multi_rhs" > gpurun_out/pytest_wave.log 2>&1; echo "pytest rc=$?"
tail -5 gpurun_out/pytest_wave.log
