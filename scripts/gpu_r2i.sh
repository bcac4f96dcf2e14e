#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2i_build.log 2>&1 || { echo BUILD FAILED; tail gpurun_out/r2i_build.log; exit 1; }
export SPTRSV_GEN_CACHE=/tmp/gencache
SPTRSV_SF_WROW=1 timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "small_configs or forced_kernels or variants or fp32 or upper or adversarial or long_chain" > gpurun_out/r2i_pytest.log 2>&1; echo "pytest wrow rc=$?"; tail -3 gpurun_out/r2i_pytest.log
echo "== WROW"
SPTRSV_SF_WROW=1 timeout 900 python scripts/sweep_sf.py C3 SPTRSV_SF_WROW_CTAS=296 SPTRSV_SF_WROW_CTAS=148 2>&1 | tail -3
echo "== MIXED"
SPTRSV_SF_MIXED=1 timeout 900 python scripts/sweep_sf.py C3 2>&1 | tail -1
SPTRSV_NVCC_FLAGS=-DSPTRSV_SF_TRACE python -c "from paper_conf_icpp_lun020_b200 import build; build.build(force=True)" > /dev/null 2>&1
mkdir -p /tmp/sft
echo "== trace WROW"; SPTRSV_SF_WROW=1 SPTRSV_SF_TRACE=/tmp/sft timeout 600 python scripts/sf_trace.py C3 2>&1 | tail -24
