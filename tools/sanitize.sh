#!/bin/bash
# compute-sanitizer over a short C1 replay (memcheck, racecheck, synccheck) on both
# transfer paths.  Output under gpurun_out/sanitize/.
O=gpurun_out/sanitize; mkdir -p $O
CS=/usr/local/cuda/bin/compute-sanitizer
cat > /tmp/san_run.py <<'PY'
import os, sys
sys.path.insert(0, os.getcwd())
import tracegen as tg
from oracle.sim import replay
from paper_conf_iiswc_zhucvhcr22_b200 import harness, um
t = tg.gen_c1(int(sys.argv[2])).slice_ops(0, int(sys.argv[3]))
flags = um.UM_F_APP_STAMP | um.UM_F_CHECK | (um.UM_F_COPY_CE if sys.argv[1] == "ce" else um.UM_F_COPY_KERNEL)
g = harness.run_trace(t, "lazy", flags=flags)
o = replay(t, "lazy").dump()
assert g["stats"] == o["stats"] and list(g["st"]) == o["st"]
print("parity ok under sanitizer", sys.argv[1:])
PY
for tool in memcheck racecheck synccheck initcheck; do
  for path in kernel ce; do
    timeout 900 $CS --tool $tool --print-limit 20 python /tmp/san_run.py $path 1 300 > $O/${tool}_${path}.log 2>&1
    echo "$tool $path rc=$? $(grep -E 'ERROR SUMMARY|RACECHECK SUMMARY|parity ok' $O/${tool}_${path}.log | tr '\n' ' ')"
  done
done
