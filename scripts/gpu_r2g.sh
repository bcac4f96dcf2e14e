#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2g_build.log 2>&1 || { echo BUILD FAILED; tail gpurun_out/r2g_build.log; exit 1; }
export SPTRSV_GEN_CACHE=/tmp/gencache
timeout 1200 python -m pytest tests/test_gpu_device_analysis.py -m gpu -q -x > gpurun_out/r2g_dev.log 2>&1; echo "dev-analysis tests rc=$?"; tail -5 gpurun_out/r2g_dev.log
SPTRSV_ANALYSE_TRACE=1 timeout 300 python scripts/time_analyse_dev.py C3 2>&1 | grep "dev\|C3" | tail -17
timeout 900 python scripts/time_analyse_dev.py C5 C2 C4 2>&1 | tail -3
SPTRSV_SF_MIXED=1 timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "small_configs or forced_kernels or variants or fp32 or upper or adversarial or long_chain" > gpurun_out/r2g_pytest.log 2>&1; echo "pytest mixed rc=$?"; tail -3 gpurun_out/r2g_pytest.log
echo "== MIXED v4"
SPTRSV_SF_MIXED=1 timeout 900 python scripts/sweep_sf.py C3 SPTRSV_SF_CTAS=148 SPTRSV_SF_CTAS=592 2>&1 | tail -3
SPTRSV_NVCC_FLAGS=-DSPTRSV_SF_TRACE python -c "from paper_conf_icpp_lun020_b200 import build; build.build(force=True)" > /dev/null 2>&1
mkdir -p /tmp/sft
echo "== trace MIXED v4"; SPTRSV_SF_MIXED=1 SPTRSV_SF_TRACE=/tmp/sft timeout 600 python scripts/sf_trace.py C3 2>&1 | tail -24
