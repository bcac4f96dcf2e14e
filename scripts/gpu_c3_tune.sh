#!/bin/bash
# C3 tuning: sync-free warp/thread threshold, row-block size of SQ_ADAPT
mkdir -p gpurun_out; export SPTRSV_GEN_CACHE=/tmp/sptrsv_gen
for thr in 8 1000; do
  SPTRSV_SF_WARP_NPR=$thr timeout 600 python scripts/time_segs.py --config C3 --tag "warp_npr=$thr" 2>&1 | tail -1
done
for nb in ${NBS:-128 512}; do
  SPTRSV_NVCC_FLAGS="-DSPTRSV_SQ_NB=$nb" python -c "from paper_conf_icpp_lun020_b200 import build; build.build(force=True)" > gpurun_out/build_exp.log 2>&1 || tail -3 gpurun_out/build_exp.log
  timeout 600 python scripts/time_segs.py --config C3 --tag "sq_nb=$nb" 2>&1 | tail -1
done
python -c "from paper_conf_icpp_lun020_b200 import build; build.build(force=True)" > /dev/null 2>&1
