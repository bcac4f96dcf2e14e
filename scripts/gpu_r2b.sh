#!/bin/bash
# round 2: boundary tests (allocator hooks, graphs, watchdog), full GPU suite, C3 bench
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/r2b_smoke.log 2>&1; echo "smoke rc=$?"; tail -2 gpurun_out/r2b_smoke.log
timeout 900 python -m pytest tests/test_gpu_boundary.py -m gpu -q > gpurun_out/r2b_boundary.log 2>&1; echo "boundary rc=$?"
tail -15 gpurun_out/r2b_boundary.log
timeout 1800 python -m pytest tests -m gpu -x -q > gpurun_out/r2b_pytest.log 2>&1; echo "pytest rc=$?"
tail -5 gpurun_out/r2b_pytest.log
timeout 600 python bench.py --steps 20 --warmup 3 --cpu-seconds 2 > gpurun_out/r2b_bench_C3.log 2>&1; echo "bench rc=$?"
tail -c 2500 gpurun_out/r2b_bench_C3.log
