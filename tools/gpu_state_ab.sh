#!/bin/bash
# A/B of an env toggle on bench.py's state microbench: VAR=name, runs 0 and 1
for v in 1 0; do
  echo "== $VAR=$v"
  env $VAR=$v timeout 300 python tools/state_bench.py --reps 3 2>&1 | python -c "
import json,sys
for l in sys.stdin:
  try: d=json.loads(l)
  except Exception: print(l[:200]); continue
  print({k:(round(v['ms']*1000,2), round(v['frac'],3)) for k,v in d.items() if isinstance(v,dict)})"
done
