#!/bin/bash
# last checks of the round: compute-sanitizer on the K4-CE path (mapped plan read-back),
# smoke, then the default bench line
O=gpurun_out/sanitize; mkdir -p $O
CS=/usr/local/cuda/bin/compute-sanitizer
cat > /tmp/san_ce.py <<'PY'
import os, sys
sys.path.insert(0, os.getcwd())
import numpy as np
import tracegen as tg
from oracle.sim import replay
from paper_conf_iiswc_zhucvhcr22_b200 import harness, um
t = tg.gen_c3(block_bytes=64 << 10, budget_bytes=192 << 20, iterations=1, workspace_bytes=4 << 20,
              layers=tg.scale_layers(tg.VGG16, 1.0 / 512, 1.0 / 64), batch=8)
g = harness.run_trace(t, "eager", flags=um.UM_F_APP_STAMP | um.UM_F_CHECK | um.UM_F_COPY_CE)
o = replay(t, "eager").dump()
assert g["stats"] == o["stats"] and list(g["st"]) == o["st"]
assert np.array_equal(np.asarray(g["contents"], np.uint64), np.asarray(o["contents"], np.uint64))
print("parity ok under sanitizer (C3-small, K4-CE)")
PY
for tool in memcheck racecheck synccheck; do
  timeout 900 $CS --tool $tool --print-limit 20 python /tmp/san_ce.py > $O/${tool}_ce_mapped.log 2>&1
  echo "${tool}_ce_mapped: rc=$? $(grep -E 'ERROR SUMMARY|RACECHECK SUMMARY|parity ok' $O/${tool}_ce_mapped.log | tr '\n' ' ')"
done
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
s=$(date +%s)
timeout 1500 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench rc=$? wall=$(( $(date +%s) - s ))s"
