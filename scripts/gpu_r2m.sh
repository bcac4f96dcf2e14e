#!/bin/bash
mkdir -p gpurun_out
export SPTRSV_GEN_CACHE=/tmp/gencache
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2m_build.log 2>&1 || { echo BUILD FAILED; tail gpurun_out/r2m_build.log; exit 1; }
echo "== fused"; timeout 600 python scripts/sweep_sf.py C3 2>&1 | tail -1
echo "== unfused"; SPTRSV_NO_SQ_FUSE=1 timeout 600 python scripts/sweep_sf.py C3 2>&1 | tail -1
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_device_analysis.py tests/test_gpu_boundary.py -m gpu -x -q > gpurun_out/r2m_pytest.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/r2m_pytest.log
