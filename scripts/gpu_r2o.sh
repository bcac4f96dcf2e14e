#!/bin/bash
mkdir -p gpurun_out
export SPTRSV_GEN_CACHE=/tmp/gencache
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2o_build.log 2>&1 || { echo BUILD FAILED; tail gpurun_out/r2o_build.log; exit 1; }
for t in 16 0 8 32; do
  echo "== C5 SPMM_TILE=$t"; SPTRSV_SPMM_TILE=$t SWEEP_NRHS=512 timeout 900 python scripts/sweep_sf.py C5 2>&1 | tail -1
done
for c in C1 C2 C4 C5; do
  timeout 900 python bench.py --config $c --steps 20 --warmup 3 --cpu-seconds 3 > gpurun_out/r2o_bench_$c.log 2>&1; echo "bench $c rc=$?"
  python - "$c" <<'PY'
import json,sys
c=sys.argv[1]
for l in open(f"gpurun_out/r2o_bench_{c}.log"):
    if l.startswith("{"):
        d=json.loads(l); print(c, "GFLOPS=%.2f ms=%.4f pre=%.1f frac=%.4f" % (d["value"], d["ms_per_step"], d["preprocess_ms"], d["roofline"]["frac"]), {k: round(v,4) for k,v in d["segment_ms"].items()}, "err", d["parity"]["rel_err"])
PY
done
timeout 1800 python -m pytest tests -m gpu -x -q > gpurun_out/r2o_pytest.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/r2o_pytest.log
