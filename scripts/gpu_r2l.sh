#!/bin/bash
mkdir -p gpurun_out
export SPTRSV_GEN_CACHE=/tmp/gencache
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2l_build.log 2>&1 || { echo BUILD FAILED; tail gpurun_out/r2l_build.log; exit 1; }
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_device_analysis.py tests/test_gpu_boundary.py -m gpu -x -q > gpurun_out/r2l_pytest.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/r2l_pytest.log
echo "== MIXED MINB3 fused"; timeout 600 python scripts/sweep_sf.py C3 2>&1 | tail -1
echo "== MIXED MINB3 unfused"; SPTRSV_NO_SQ_FUSE=1 timeout 600 python scripts/sweep_sf.py C3 2>&1 | tail -1
SPTRSV_NVCC_FLAGS="-DSPTRSV_SFM_MINB=2" python -c "from paper_conf_icpp_lun020_b200 import build; build.build(force=True)" > /dev/null 2>&1
echo "== MIXED MINB2 fused"; timeout 600 python scripts/sweep_sf.py C3 SPTRSV_SF_CTAS=296 2>&1 | tail -2
echo "== MIXED MINB2 unfused"; SPTRSV_NO_SQ_FUSE=1 timeout 600 python scripts/sweep_sf.py C3 2>&1 | tail -1
