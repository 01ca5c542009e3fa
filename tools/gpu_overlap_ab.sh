#!/bin/bash
# A/B of the R7 overlap: app CTAs per SM (UM_APP_CTAS), C3 bench without the side measurements
mkdir -p gpurun_out
for c in ${CTAS:-1 2}; do
  UM_APP_CTAS=$c timeout 900 python bench.py --no-discard-bench --no-state-bench --no-e2e --no-cpu \
    > gpurun_out/bench_ab_$c.json 2> gpurun_out/bench_ab_$c.err; echo "ctas=$c rc=$?"
  python - $c <<'PY'
import json, sys
d = json.loads(open(f"gpurun_out/bench_ab_{sys.argv[1]}.json").read().strip().splitlines()[-1])
print(sys.argv[1], {k: d.get(k) for k in ("iter_ms", "app_overlap", "plan_ms_per_iter")}, d["roofline"]["xfer_share_of_step"])
PY
done
