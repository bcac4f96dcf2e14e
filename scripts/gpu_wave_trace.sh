#!/bin/bash
# Instrumented build (per-group globaltimer stamps in tri_wave), C2 trace dump.
mkdir -p gpurun_out/tr
SPTRSV_NVCC_FLAGS="-DSPTRSV_WAVE_TRACE" python -c "from paper_conf_icpp_lun020_b200 import build; build.build(force=True)" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
SPTRSV_TRACE=1 SPTRSV_TRACE_DIR=gpurun_out/tr timeout 300 python scripts/prof_solve.py --config C2 --reps 3 > gpurun_out/trace.log 2>&1; echo "trace rc=$?"
ls -la gpurun_out/tr
python -c "from paper_conf_icpp_lun020_b200 import build; build.build(force=True)" > /dev/null 2>&1
