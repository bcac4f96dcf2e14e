#!/bin/bash
# wave kernel iteration: parity subset, isolated loop time, C2 bench
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "TRI_PIPE or wave or small_configs" > gpurun_out/pytest_wave.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pytest_wave.log
SPTRSV_WAVE=1,1,12,4 timeout 120 python scripts/wave_iso.py --tag "iso" 2>&1 | tail -1
CONFIGS="C2" bash scripts/gpu_iter.sh
