#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2h_build.log 2>&1 || { echo BUILD FAILED; tail gpurun_out/r2h_build.log; exit 1; }
nvcc -gencode arch=compute_100a,code=sm_100a -O3 scripts/microbench/hop_load.cu -o /tmp/hop_load && timeout 300 /tmp/hop_load
export SPTRSV_GEN_CACHE=/tmp/gencache
timeout 1200 python -m pytest tests/test_gpu_device_analysis.py -m gpu -q > gpurun_out/r2h_dev.log 2>&1; echo "dev-analysis tests rc=$?"; tail -3 gpurun_out/r2h_dev.log
SPTRSV_ANALYSE_TRACE=1 timeout 600 python scripts/time_analyse_dev.py C3 C2 2>&1 | grep "dev:\|wave\|C3\|C2" | tail -40
