#!/bin/bash
# C5 bisect over round-2 commits; cluster level-set experiment on C3
O=gpurun_out/r2s
mkdir -p $O
export SPTRSV_GEN_CACHE=/tmp/gencache
summ() { python - "$1" <<'PY'
import json,sys
for l in open(sys.argv[1]):
    if l.startswith("{"):
        d=json.loads(l); print(sys.argv[1].split('/')[-1], "ms=%.4f" % d["ms_per_step"], {k: round(v,3) for k,v in d.get("segment_ms",{}).items()})
PY
}
for c in bdf3ee8 2dade3b 0032d24; do
(cd _w$c && timeout 900 python bench.py --config C5 --steps 5 --warmup 3 --no-cpu-baseline > ../$O/bench_$c.log 2>&1); echo "$c rc=$?"; summ $O/bench_$c.log
done
SPTRSV_SF_CLUSTER=16 timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "test_forced_kernels and TRI_SYNCFREE and SQ_ADAPT" > $O/cl_pytest.log 2>&1; echo "cluster pytest rc=$?"; tail -3 $O/cl_pytest.log
timeout 600 python scripts/sweep_sf.py C3 2>&1 | tail -1
for cs in 16 8 4; do echo "== cluster $cs"; SPTRSV_SF_CLUSTER=$cs timeout 600 python scripts/sweep_sf.py C3 2>&1 | tail -2; done
