#!/bin/bash
# compute-sanitizer (memcheck, racecheck, synccheck) over short traces on every path:
# single-level K4, copy-engine arm, two-level pages (+ free), device-resident records with
# proactive eviction, with parity asserted under
# the tool.  Output under gpurun_out/sanitize/.
O=gpurun_out/sanitize; mkdir -p $O
CS=/usr/local/cuda/bin/compute-sanitizer
cat > /tmp/san_run.py <<'PY'
import os, sys
sys.path.insert(0, os.getcwd())
sys.path.insert(0, os.path.join(os.getcwd(), "tests"))
import numpy as np
import tracegen as tg
from oracle.sim import replay
from oracle.chunks import replay_chunks
from paper_conf_iiswc_zhucvhcr22_b200 import harness, um
what = sys.argv[1]
if what == "devrec":
    # device-resident records (k_mark_acc, k_list) incl. unsorted batches, and proactive
    # eviction (R12) through the evict-mode victim path
    t = tg.gen_random(3, block_bytes=64 << 10, arena_bytes=32 << 20, budget_bytes=4 << 20, n_ops=150,
                      max_ranges=200, max_blocks=8, zipf_s=0.8)
    g = harness.run_trace(t, "eager", flags=um.UM_F_APP_STAMP | um.UM_F_CHECK, dev_records=True, reserve_blocks=4,
                          xlog=1 << 18)
    o = replay(t, "eager", reserve=4, record=True)
    assert g["stats"] == o.dump()["stats"] and list(g["st"]) == o.dump()["st"] and g["xlog"] == sorted(o.log)
elif what in ("kernel", "ce"):
    t = tg.gen_c1(1).slice_ops(0, 300)
    flags = um.UM_F_APP_STAMP | um.UM_F_CHECK | (um.UM_F_COPY_CE if what == "ce" else 0)
    g = harness.run_trace(t, "lazy", flags=flags, xlog=1 << 16)
    o = replay(t, "lazy", record=True)
    assert g["stats"] == o.dump()["stats"] and list(g["st"]) == o.dump()["st"] and g["xlog"] == sorted(o.log)
else:
    from test_gpu_pages import _random_page_trace
    t = _random_page_trace(3, 64 << 10, 32, 5, 2, n_ops=40)
    t2 = tg.gen_hashjoin(block_bytes=64 << 10, budget_bytes=(24 << 20), table_bytes=4 << 20, free_at_end=True)
    g = harness.run_trace(t, "eager", page_bytes=64 << 10, flags=um.UM_F_APP_STAMP | um.UM_F_CHECK, xlog=1 << 16)
    o = replay_chunks(t, 64 << 10, "eager", record=True)
    assert g["stats"] == o.dump()["stats"] and g["xlog"] == sorted(o.log)
    assert np.array_equal(np.asarray(g["contents"], np.uint64), np.asarray(o.contents(), np.uint64))
    g = harness.run_trace(t2, "eager", flags=um.UM_F_APP_STAMP | um.UM_F_CHECK)
    assert g["stats"] == replay(t2, "eager").dump()["stats"]
print("parity ok under sanitizer", what)
PY
for tool in memcheck racecheck synccheck; do
  for path in kernel ce pages devrec; do
    timeout 600 $CS --tool $tool --print-limit 20 python /tmp/san_run.py $path > $O/${tool}_${path}.log 2>&1
    echo "$tool $path rc=$? $(grep -E 'ERROR SUMMARY|RACECHECK SUMMARY|parity ok' $O/${tool}_${path}.log | tr '\n' ' ')"
  done
done
