#!/bin/bash
# Focused check of the strand wavefront kernel: build, wave tests, C2 bench.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "wave or forced_kernels or multi_rhs" ${PYTEST_ARGS} > gpurun_out/pytest_wave.log 2>&1; echo "pytest rc=$?"
tail -30 gpurun_out/pytest_wave.log
timeout 300 python bench.py --config C2 --steps 30 --warmup 3 --no-cpu-baseline > gpurun_out/bench_C2.log 2>&1; echo "bench rc=$?"
grep '^{' gpurun_out/bench_C2.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['ms_per_step'], d['segment_ms'], d['roofline'])"
tail -3 gpurun_out/bench_C2.log
