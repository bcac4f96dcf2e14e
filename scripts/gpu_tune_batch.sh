#!/bin/bash
export SPTRSV_GEN_CACHE=/tmp/sptrsv_gen
mkdir -p gpurun_out
for c in C1 C3 C5; do
  SPTRSV_ANALYSE_TRACE=1 timeout 600 python /root/repo/scripts/time_analyse.py $c 2>&1 | tail -16
done
bash scripts/gpu_c3_tune.sh
bash scripts/gpu_c4_tune.sh
