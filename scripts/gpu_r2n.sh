#!/bin/bash
mkdir -p gpurun_out
export SPTRSV_GEN_CACHE=/tmp/gencache
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2n_build.log 2>&1 || { echo BUILD FAILED; tail gpurun_out/r2n_build.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "supernode or C4" > gpurun_out/r2n_sn.log 2>&1; echo "sn tests rc=$?"; tail -2 gpurun_out/r2n_sn.log
echo "== C4 split"; timeout 600 python scripts/sweep_sf.py C4 2>&1 | tail -1
echo "== C4 nosplit"; SPTRSV_SN_NOSPLIT=1 timeout 600 python scripts/sweep_sf.py C4 2>&1 | tail -1
timeout 1200 python -m pytest tests/test_gpu_dist.py -m gpu -q > gpurun_out/r2n_dist.log 2>&1; echo "dist rc=$?"; tail -3 gpurun_out/r2n_dist.log
SPTRSV_ANALYSE_TRACE=1 timeout 300 python scripts/time_analyse_dev.py C3 2>&1 | grep "dev:\|C3" | tail -14
timeout 900 python bench.py --steps 20 --warmup 3 --cpu-seconds 3 > gpurun_out/r2n_bench_C3.log 2>&1; echo "bench rc=$?"; tail -c 1500 gpurun_out/r2n_bench_C3.log
timeout 1500 python scripts/fig5_derive.py --quick > gpurun_out/r2n_fig5.log 2>&1; echo "fig5 rc=$?"; tail -8 gpurun_out/r2n_fig5.log
cp profiles/r02_fig5.json gpurun_out/ 2>/dev/null
