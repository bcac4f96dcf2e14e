#!/bin/bash
# round 2: full-size multi-RHS parity on every column + C3 bench baseline
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 1500 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "all_columns or full_size_configs" > gpurun_out/r2a_pytest.log 2>&1; echo "pytest rc=$?"
tail -3 gpurun_out/r2a_pytest.log
timeout 600 python bench.py --config C3 --steps 20 --warmup 3 --cpu-seconds 2 > gpurun_out/r2a_bench_C3.log 2>&1; echo "bench rc=$?"
tail -c 3000 gpurun_out/r2a_bench_C3.log
nproc; lscpu | grep "Model name"
