#!/bin/bash
# after the warp-uniform watchdog fix: full GPU suite, watchdog test x5 in a busy process, C3/C4/C5 bench lines
O=gpurun_out/r2final4
mkdir -p $O
export SPTRSV_GEN_CACHE=/tmp/gencache
timeout 2400 python -m pytest tests -m gpu -q > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -2 $O/pytest_gpu.log
timeout 900 python -m pytest tests/test_gpu_boundary.py tests/test_gpu_parity.py -q -k "watchdog or small_configs" --count 1 > /dev/null 2>&1
for i in 1 2 3; do timeout 400 python -m pytest tests/test_gpu_boundary.py -q -k watchdog 2>&1 | tail -1; done
summ() { python - "$1" <<'PY'
import json,sys
for l in open(sys.argv[1]):
    if l.startswith("{"):
        d=json.loads(l); print(sys.argv[1].split('/')[-1], "ms=%.4f GFLOPS=%.2f frac=%.4f" % (d["ms_per_step"], d["value"], d["roofline"]["frac"]), d["roofline"].get("kernel"), "pre=%.1f" % d["preprocess_ms"], "e2e=%.2f" % d["e2e"]["value"], "err", d["parity"]["rel_err"])
PY
}
for c in C3 C4 C5 C2 C1; do steps=20; [ $c = C5 ] && steps=5
timeout 900 python bench.py --config $c --steps $steps --warmup 3 --cpu-seconds 10 > $O/bench_$c.log 2>&1; echo "$c rc=$?"; summ $O/bench_$c.log; done
