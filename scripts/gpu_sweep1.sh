#!/bin/bash
# chain v2 parity + C2 bench; SpMM variant sweep on C5; backoff / CTA sweep on C3, C4
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?"; tail -1 gpurun_out/smoke.log
timeout 900 python -m pytest tests -m gpu -x -q -k "C2 or chain or CHAIN or adversarial or fp32 or upper" > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -4 gpurun_out/pytest_gpu.log
summ() { python - "$1" <<'PY'
import json,sys
for l in open(sys.argv[1]):
    if l.startswith("{"):
        d=json.loads(l); print("GFLOPS=%.3f ms=%.4f" % (d["value"], d["ms_per_step"]), {k: round(v,4) for k,v in d["segment_ms"].items()}, "err", d["parity"]["rel_err"])
PY
}
timeout 600 python bench.py --config C2 --steps 20 --warmup 3 --no-cpu-baseline > gpurun_out/bench_C2.log 2>&1; echo "C2 rc=$?"; summ gpurun_out/bench_C2.log
SPTRSV_TRACE=1 python scripts/prof_solve.py --config C2 --reps 2 2>&1 | grep trace | tail -2
for w in 4 8 12; do echo "warps $w"; SPTRSV_ELL_WARPS=$w timeout 600 python bench.py --config C2 --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/b.log 2>&1; summ gpurun_out/b.log; done
for v in 16,1 8,1 8,2 4,2 4,1; do echo "SPMM $v"; SPTRSV_SPMM=$v timeout 600 python bench.py --config C5 --steps 3 --warmup 2 --no-cpu-baseline > gpurun_out/b.log 2>&1; summ gpurun_out/b.log; done
for c in C3 C4; do for bo in 0 64 128 256; do echo "$c backoff $bo"; SPTRSV_SF_BACKOFF=$bo timeout 600 python bench.py --config $c --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/b.log 2>&1; summ gpurun_out/b.log; done; done
for c in C3 C4; do for ct in 592 1184; do echo "$c ctas $ct"; SPTRSV_SF_CTAS=$ct timeout 600 python bench.py --config $c --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/b.log 2>&1; summ gpurun_out/b.log; done; done
