#!/bin/bash
# round-2 fixes: C5 seg0 predicate fix + untiled SpMM default, persistent sq_adapt_1 (C3 squares)
O=gpurun_out/r2u
mkdir -p $O
export SPTRSV_GEN_CACHE=/tmp/gencache
summ() { python - "$1" <<'PY'
import json,sys
for l in open(sys.argv[1]):
    if l.startswith("{"):
        d=json.loads(l); print(sys.argv[1].split('/')[-1], "ms=%.4f GFLOPS=%.2f frac=%.4f" % (d["ms_per_step"], d["value"], d["roofline"]["frac"]), {k: round(v,3) for k,v in d.get("segment_ms",{}).items()})
PY
}
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "forced_kernels or multi_rhs or square_row_blocks" > $O/pytest.log 2>&1; echo "pytest rc=$?"; tail -2 $O/pytest.log
for c in C5 C3; do
timeout 900 python bench.py --config $c --steps 10 --warmup 3 --no-cpu-baseline > $O/bench_$c.log 2>&1; echo "$c rc=$?"; summ $O/bench_$c.log
done
for n in 2 3 4 6; do echo "== SQ_CTAS=$n"; SPTRSV_SQ_CTAS=$n timeout 600 python scripts/sweep_sf.py C3 2>&1 | tail -1; done
