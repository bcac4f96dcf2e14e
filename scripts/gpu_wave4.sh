#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
timeout 300 python scripts/time_segs.py --config C2 --tag "default" 2>&1 | tail -1
for geo in "8,4,12,4" "16,2,12,4" "16,4,6,4" "16,4,12,3"; do
  SPTRSV_WAVE=$geo timeout 300 python scripts/time_segs.py --config C2 --tag "geo=$geo" 2>&1 | tail -1
done
mkdir -p gpurun_out/tr
true
timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "wave or forced_kernels or multi_rhs" > gpurun_out/pytest_wave.log 2>&1; echo "pytest rc=$?"
tail -5 gpurun_out/pytest_wave.log
