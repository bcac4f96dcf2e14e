#!/bin/bash
# bench after the clock-sampler move: C1, C2, default (C3)
export SPTRSV_GEN_CACHE=/tmp/gencache
O=gpurun_out/r2bench
mkdir -p $O
for c in C1 C2; do timeout 600 python bench.py --config $c --steps 20 --warmup 3 --cpu-seconds 3 > $O/bench_$c.log 2>&1; echo "$c rc=$?"; done
timeout 900 python bench.py > $O/bench_default.log 2>&1; echo "default rc=$?"
python - <<'PY'
import json, glob
for f in sorted(glob.glob("gpurun_out/r2bench/*.log")):
    for l in open(f):
        if l.startswith("{"):
            d = json.loads(l); t = d["timing"]
            print(f.split("/")[-1], "ms=%.4f mean=%.4f median=%.4f p90=%.4f" % (d["ms_per_step"], t["mean_ms"], t["median_ms"], t["p90_ms"]), "clocks", d["clocks"], "steps", d["steps"], d["config"]["workload"][:20])
PY
