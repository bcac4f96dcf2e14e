#!/bin/bash
# C5 regression bisect: round-1 tree (_r1) vs HEAD, tiled vs untiled SpMM, host vs device analysis
O=gpurun_out/r2q
mkdir -p $O
export SPTRSV_GEN_CACHE=/tmp/gencache
summ() { python - "$1" <<'PY'
import json,sys
for l in open(sys.argv[1]):
    if l.startswith("{"):
        d=json.loads(l); print(sys.argv[1].split('/')[-1], "ms=%.4f" % d["ms_per_step"], {k: round(v,3) for k,v in d.get("segment_ms",{}).items()})
PY
}
(cd _r1 && timeout 900 python bench.py --config C5 --steps 5 --warmup 3 --no-cpu-baseline > ../$O/bench_r1.log 2>&1); echo "r1 rc=$?"; summ $O/bench_r1.log
SPTRSV_SPMM_TILE=0 timeout 900 python bench.py --config C5 --steps 5 --warmup 3 --no-cpu-baseline > $O/bench_t0.log 2>&1; echo "t0 rc=$?"; summ $O/bench_t0.log
SWEEP_NRHS=512 timeout 900 python scripts/sweep_sf.py C5 SPTRSV_SPMM_TILE=0 SPTRSV_SPMM_TILE=8 SPTRSV_SPMM_TILE=32 2>&1 | tail -4
