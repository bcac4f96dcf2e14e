#!/bin/bash
# chain v2 + supernodal parity, C2/C4 bench, sync-free grid sweep on C3
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?"; tail -3 gpurun_out/smoke.log
timeout 900 python -m pytest tests -m gpu -x -q -k "C2 or C4 or chain or CHAIN or adversarial or fp32 or upper" > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -4 gpurun_out/pytest_gpu.log
summ() { python - "$1" <<'PY'
import json,sys
for l in open(sys.argv[1]):
    if l.startswith("{"):
        d=json.loads(l); print("GFLOPS=%.3f ms=%.4f" % (d["value"], d["ms_per_step"]), {k: round(v,4) for k,v in d["segment_ms"].items()}, "err", d["parity"]["rel_err"])
PY
}
timeout 300 python bench.py --config C2 --steps 20 --warmup 3 --no-cpu-baseline > gpurun_out/bench_C2.log 2>&1; echo "C2 rc=$?"; summ gpurun_out/bench_C2.log; tail -2 gpurun_out/bench_C2.log | cut -c1-300
SPTRSV_TRACE=1 timeout 120 python scripts/prof_solve.py --config C2 --reps 2 2>&1 | grep trace | tail -2
for w in 4 8 12 16; do echo "warps $w"; SPTRSV_ELL_WARPS=$w timeout 300 python bench.py --config C2 --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/b.log 2>&1; summ gpurun_out/b.log; done
timeout 300 python bench.py --config C4 --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/bench_C4.log 2>&1; echo "C4 rc=$?"; summ gpurun_out/bench_C4.log; tail -2 gpurun_out/bench_C4.log | cut -c1-300
for ct in 148 296 444; do echo "C3 ctas $ct"; SPTRSV_SF_CTAS=$ct timeout 300 python bench.py --config C3 --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/b.log 2>&1; summ gpurun_out/b.log; done
