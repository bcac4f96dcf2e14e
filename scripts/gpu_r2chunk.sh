#!/bin/bash
# supernode chunk-width sweep (C4 forward, one RHS); rebuilds per width
export SPTRSV_GEN_CACHE=/tmp/gencache
for w in 64 128 256 512; do
  SPTRSV_NVCC_FLAGS=-DSPTRSV_SN_CHUNK=$w python -c "import __graft_entry__ as g; g.build()" > /tmp/b.log 2>&1 || { echo "build $w failed"; tail -3 /tmp/b.log; continue; }
  echo "== chunk $w"; timeout 600 python scripts/depth_probe.py C4 0 2>&1 | grep depth
done
python -c "import __graft_entry__ as g; g.build()" > /tmp/b.log 2>&1
