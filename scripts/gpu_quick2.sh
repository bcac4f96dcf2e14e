#!/bin/bash
# quick GPU iteration: build, GPU parity tests (optional -k filter), benches
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?"; tail -1 gpurun_out/smoke.log
if [ -z "$NO_TEST" ]; then
timeout ${TEST_TIMEOUT:-1200} python -m pytest tests -m gpu -x -q ${PYTEST_K:+-k "$PYTEST_K"} > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -4 gpurun_out/pytest_gpu.log
fi
for c in ${CONFIGS:-C2}; do
  steps=20; [ $c = C5 ] && steps=5
  timeout 900 python bench.py --config $c --steps $steps --warmup 3 --no-cpu-baseline ${BENCH_ARGS} > gpurun_out/bench_$c.log 2>&1; echo "bench $c rc=$?"
  python - "$c" <<'PY'
import json,sys
c=sys.argv[1]
for l in open(f"gpurun_out/bench_{c}.log"):
    if l.startswith("{"):
        d=json.loads(l); print(c, "GFLOPS=%.3f ms=%.4f frac=%.4f" % (d["value"], d["ms_per_step"], d["roofline"]["frac"]), {k: round(v,4) for k,v in d["segment_ms"].items()}, "err", d["parity"]["rel_err"])
PY
done
