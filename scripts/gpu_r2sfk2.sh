#!/bin/bash
# tri_sf_mixed: long-row threshold x batch size on C3 (depth 1) and C5 (one RHS)
export SPTRSV_GEN_CACHE=/tmp/gencache
for f in "-DSPTRSV_SF_LONG=64" "-DSPTRSV_SF_LONG=96" "-DSPTRSV_SF_LONG=128" "-DSPTRSV_SF_LONG=64 -DSPTRSV_SF_U=8" "-DSPTRSV_SF_LONG=128 -DSPTRSV_SF_U=8"; do
  SPTRSV_NVCC_FLAGS="$f" python -c "import __graft_entry__ as g; g.build()" > /tmp/b.log 2>&1 || { echo "build '$f' failed"; tail -3 /tmp/b.log; continue; }
  echo "== flags '$f'"; timeout 600 python scripts/sweep_sf.py C3 2>&1 | tail -1; timeout 600 python scripts/depth_probe.py C5 0 2>&1 | grep depth
done
python -c "import __graft_entry__ as g; g.build()" > /tmp/b.log 2>&1
