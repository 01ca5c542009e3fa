#!/bin/bash
# A/B of env settings on bench.py's state microbench: CONFIGS="A=1 B=2;A=0" (';'-separated)
IFS=';' read -ra CFG <<< "${CONFIGS:-X=0}"
for c in "${CFG[@]}"; do
  echo "== $c"
  env $c timeout 300 python tools/state_bench.py --reps 3 2>&1 | python -c "
import json,sys
for l in sys.stdin:
  try: d=json.loads(l)
  except Exception: print(l[:200]); continue
  print({k:(round(v['ms']*1000,2), round(v['frac'],3)) for k,v in d.items() if isinstance(v,dict)})"
done
