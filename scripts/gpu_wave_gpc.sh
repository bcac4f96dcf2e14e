#!/bin/bash
# wave: parity subset + C2 timing at GPC 12 (default build) and 24
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "TRI_PIPE or wave or small_configs" > gpurun_out/pytest_wave.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pytest_wave.log
timeout 300 python scripts/time_segs.py --config C2 --tag "gpc=12" 2>&1 | tail -1
SPTRSV_WAVE=1,1,12,4 timeout 120 python scripts/wave_iso.py --tag "iso gpc=12" 2>&1 | tail -1
for G in ${GPCS:-24}; do
SPTRSV_NVCC_FLAGS="-DSPTRSV_WAVE_GPC_BIG=$G" python -c "from paper_conf_icpp_lun020_b200 import build; build.build(force=True)" > gpurun_out/build_exp.log 2>&1 || tail -3 gpurun_out/build_exp.log
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "TRI_PIPE or wave" > gpurun_out/pytest_wave24.log 2>&1; echo "pytest gpc=$G rc=$?"; tail -1 gpurun_out/pytest_wave24.log
timeout 300 python scripts/time_segs.py --config C2 --tag "gpc=$G" 2>&1 | tail -1
SPTRSV_WAVE=1,1,12,4 timeout 120 python scripts/wave_iso.py --tag "iso gpc=$G" 2>&1 | tail -1
done
python -c "from paper_conf_icpp_lun020_b200 import build; build.build(force=True)" > /dev/null 2>&1
