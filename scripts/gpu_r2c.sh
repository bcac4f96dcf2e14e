#!/bin/bash
# round 2: row-block sync-free kernel (SPTRSV_SF_ITEMS) parity + C3 timing + per-level traces
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
export SPTRSV_GEN_CACHE=/tmp/gencache
SPTRSV_SF_ITEMS=1 timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "small_configs or forced_kernels or variants or fp32 or upper or adversarial or long_chain or (full_size_configs and C3)" > gpurun_out/r2c_pytest.log 2>&1; echo "pytest items rc=$?"; tail -3 gpurun_out/r2c_pytest.log
for v in "" "SPTRSV_SF_ITEMS=1" "SPTRSV_SF_ITEMS=1 SPTRSV_SF_PERSM=1" "SPTRSV_SF_ITEMS=1 SPTRSV_SF_BACKOFF=0" "SPTRSV_SF_ITEMS=1 SPTRSV_SF_BACKOFF=32"; do
  env $v timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/r2c_b.log 2>&1
  python - "$v" <<'PY'
import json,sys
for l in open("gpurun_out/r2c_b.log"):
    if l.startswith("{"):
        d=json.loads(l); print(sys.argv[1] or "V1", "ms=%.4f" % d["ms_per_step"], {k: round(v,3) for k,v in d["segment_ms"].items()}, "err", d["parity"]["rel_err"])
PY
done
SPTRSV_NVCC_FLAGS=-DSPTRSV_SF_TRACE python -c "from paper_conf_icpp_lun020_b200 import build; build.build(force=True)" > /dev/null 2>&1
mkdir -p /tmp/sft
echo "== trace V1"; SPTRSV_SF_TRACE=/tmp/sft timeout 600 python scripts/sf_trace.py C3 2>&1 | tail -40
echo "== trace ITEMS"; SPTRSV_SF_ITEMS=1 SPTRSV_SF_TRACE=/tmp/sft timeout 600 python scripts/sf_trace.py C3 2>&1 | tail -40
