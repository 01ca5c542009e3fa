#!/bin/bash
# compute-sanitizer over the multi-CTA state path (k_classify, k_victims_scan/apply,
# k_directive on large ranges): the wide-victim parity trace of tests/test_gpu_parity.py,
# both transfer paths.  Output under gpurun_out/sanitize/.
O=gpurun_out/sanitize; mkdir -p $O
CS=/usr/local/cuda/bin/compute-sanitizer
cat > /tmp/san_wide.py <<'PY'
import os, sys
sys.path.insert(0, os.getcwd())
import tracegen as tg
from oracle.sim import replay
from paper_conf_iiswc_zhucvhcr22_b200 import harness, um
B = 4096
n_ops = int(sys.argv[2])
base = tg.gen_random(7, block_bytes=B, arena_bytes=60000 * B, budget_bytes=20000 * B, n_ops=n_ops,
                     max_ranges=3, max_blocks=14000, zipf_s=0.3, mix=[50, 20, 5, 10, 10, 0, 5])
tb = tg.TraceBuilder(B, 60000 * B, 20000 * B)
for i, (o, fl, off, ln, accs) in enumerate(base.iter_ops()):
    if o == tg.OP_TOUCH: tb.touch(accs)
    elif o == tg.OP_PREFETCH: tb.prefetch(off, ln, fl)
    elif o == tg.OP_DISCARD: tb.discard(off, ln, lazy_ok=bool(fl & 1))
    elif o == tg.OP_HOST_WRITE: tb.host_write(off, ln)
    if i % 17 == 16: tb.evict(12000 * B)
t = tb.build()
flags = um.UM_F_APP_STAMP | um.UM_F_CHECK | (um.UM_F_COPY_CE if sys.argv[1] == "ce" else um.UM_F_COPY_KERNEL)
g = harness.run_trace(t, "eager", flags=flags)
o = replay(t, "eager").dump()
assert g["stats"] == o["stats"] and list(g["st"]) == o["st"]
assert g["used_order"] == o["used_order"] and g["disc_order"] == o["disc_order"]
print("wide parity ok under sanitizer", sys.argv[1:])
PY
for tool in memcheck synccheck racecheck; do
  for path in kernel ce; do
    timeout 900 $CS --tool $tool --print-limit 20 python /tmp/san_wide.py $path ${NOPS:-40} > $O/wide_${tool}_${path}.log 2>&1
    echo "$tool $path rc=$? $(grep -E 'ERROR SUMMARY|RACECHECK SUMMARY|parity ok' $O/wide_${tool}_${path}.log | tr '\n' ' ')"
  done
done
