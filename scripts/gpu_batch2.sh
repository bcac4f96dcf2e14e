#!/bin/bash
export SPTRSV_GEN_CACHE=/tmp/sptrsv_gen
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "TRI_PIPE or wave or small_configs or host_pointers" > gpurun_out/pytest_b2.log 2>&1; echo "pytest rc=$?"; tail -1 gpurun_out/pytest_b2.log
timeout 300 python scripts/time_segs.py --config C2 --tag "Q=2" 2>&1 | tail -1
for c in C1 C3 C5; do
  SPTRSV_ANALYSE_TRACE=1 timeout 600 python scripts/time_analyse.py $c 2>&1 | grep -E "capi|depth|H2D|analyse ms" | tail -8
done
timeout 300 python scripts/time_segs.py --config C4 --tag "C4 minb=2" 2>&1 | tail -1
for q in 1 3; do
  SPTRSV_NVCC_FLAGS="-DSPTRSV_WAVE_Q=$q" python -c "from paper_conf_icpp_lun020_b200 import build; build.build(force=True)" > gpurun_out/build_exp.log 2>&1 || tail -3 gpurun_out/build_exp.log
  timeout 300 python scripts/time_segs.py --config C2 --tag "Q=$q" 2>&1 | tail -1
done
python -c "from paper_conf_icpp_lun020_b200 import build; build.build(force=True)" > /dev/null 2>&1
