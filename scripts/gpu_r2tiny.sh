#!/bin/bash
# one-launch tiny plans (C1), cluster experiment test, boundary tests
O=gpurun_out/r2tiny
mkdir -p $O
export SPTRSV_GEN_CACHE=/tmp/gencache
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_boundary.py -q -x -k "tiny or cluster or small_configs or adversarial or C1 or graph or watchdog or layouts" > $O/pytest.log 2>&1; echo "pytest rc=$?"; tail -2 $O/pytest.log
timeout 600 python bench.py --config C1 --steps 50 --warmup 5 --cpu-seconds 3 > $O/bench_C1.log 2>&1; echo "C1 rc=$?"; grep -o '"ms_per_step": [0-9.]*\|"median_ms": [0-9.]*\|"gpu_launches": [0-9]*' $O/bench_C1.log
SPTRSV_NO_TINY=1 timeout 600 python bench.py --config C1 --steps 50 --warmup 5 --no-cpu-baseline > $O/bench_C1_notiny.log 2>&1; echo "C1 notiny rc=$?"; grep -o '"ms_per_step": [0-9.]*\|"median_ms": [0-9.]*' $O/bench_C1_notiny.log
python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
