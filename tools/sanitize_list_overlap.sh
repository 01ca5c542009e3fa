#!/bin/bash
# compute-sanitizer over the fault-list form (sparse sorted batches) and the R7 overlap
# schedule (app kernels on their own stream).  Output under gpurun_out/sanitize/.
O=gpurun_out/sanitize; mkdir -p $O
CS=/usr/local/cuda/bin/compute-sanitizer
cat > /tmp/san_lo.py <<'PY'
import os, sys
sys.path.insert(0, os.getcwd())
import numpy as np
import tracegen as tg
from oracle.sim import replay
from paper_conf_iiswc_zhucvhcr22_b200 import harness, um
which = sys.argv[1]
if which == "list":
    t = tg.gen_sparse(0, nblocks=1 << 14, nframes=1 << 12, n_ops=10, max_batch=9000)
    flags, ov = um.UM_F_APP_STAMP | um.UM_F_CHECK, 0
else:
    t = tg.gen_c1(2).slice_ops(0, 300)
    flags, ov = um.UM_F_APP_STAMP | um.UM_F_CHECK | um.UM_F_OVERLAP, 2
g = harness.run_trace(t, "eager", flags=flags)
o = replay(t, "eager", overlap=ov).dump()
assert g["stats"] == o["stats"] and list(g["st"]) == o["st"]
assert np.array_equal(np.asarray(g["contents"], np.uint64), np.asarray(o["contents"], np.uint64))
print("parity ok under sanitizer", which)
PY
for tool in memcheck racecheck synccheck; do
  for w in list overlap; do
    timeout 900 $CS --tool $tool --print-limit 20 python /tmp/san_lo.py $w > $O/${tool}_${w}.log 2>&1
    echo "${tool}_${w}: rc=$? $(grep -E 'ERROR SUMMARY|RACECHECK SUMMARY|parity ok' $O/${tool}_${w}.log | tr '\n' ' ')"
  done
done
