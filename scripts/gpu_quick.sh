#!/bin/bash
# quick GPU iteration: targeted tests + bench lines for several configs
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?"
timeout ${TEST_TIMEOUT:-900} python -m pytest tests -m gpu -x -q ${PYTEST_ARGS} > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"
tail -3 gpurun_out/pytest_gpu.log
for c in ${CONFIGS:-C2}; do
  timeout 600 python bench.py --config $c --steps 20 --warmup 3 --cpu-seconds 2 ${BENCH_ARGS} > gpurun_out/bench_$c.log 2>&1; echo "bench $c rc=$?"
  python - "$c" <<'PY'
import json,sys
c=sys.argv[1]
for l in open(f"gpurun_out/bench_{c}.log"):
    if l.startswith("{"):
        d=json.loads(l); print(c, "GFLOPS=%.3f ms=%.4f pre=%.1f frac=%.4f" % (d["value"], d["ms_per_step"], d["preprocess_ms"], d["roofline"]["frac"]), {k: round(v,4) for k,v in d["segment_ms"].items()}, "err", d["parity"]["rel_err"])
PY
done
