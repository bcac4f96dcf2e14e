#!/bin/bash
# time the isolated wavefront loop with parts of it compiled out
mkdir -p gpurun_out
for x in ${EXPS:-0 1 2 4 8 16 31}; do
  SPTRSV_NVCC_FLAGS="-DSPTRSV_WAVE_EXP=$x" python -c "from paper_conf_icpp_lun020_b200 import build; build.build(force=True)" > gpurun_out/build_exp.log 2>&1 || { tail -5 gpurun_out/build_exp.log; continue; }
  SPTRSV_WAVE=1,1,12,4 timeout 120 python scripts/wave_iso.py --tag "exp=$x" 2>&1 | tail -1
done
python -c "from paper_conf_icpp_lun020_b200 import build; build.build(force=True)" > /dev/null 2>&1
