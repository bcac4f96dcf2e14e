#!/bin/bash
# C4 tuning: supernodal kernel occupancy (min CTAs/SM) and grid size
mkdir -p gpurun_out; export SPTRSV_GEN_CACHE=/tmp/sptrsv_gen
timeout 600 python scripts/time_segs.py --config C4 --tag "minb=1" 2>&1 | tail -1
for mb in ${MINBS:-2 3}; do
  SPTRSV_NVCC_FLAGS="-DSPTRSV_SN_MINB=$mb" python -c "from paper_conf_icpp_lun020_b200 import build; build.build(force=True)" > gpurun_out/build_exp.log 2>&1 || tail -3 gpurun_out/build_exp.log
  timeout 600 python scripts/time_segs.py --config C4 --tag "minb=$mb" 2>&1 | tail -1
done
python -c "from paper_conf_icpp_lun020_b200 import build; build.build(force=True)" > /dev/null 2>&1
