#!/bin/bash
mkdir -p gpurun_out
for g in 8 16 32 74; do
  echo "UM_APP_GRID=$g"
  UM_APP_GRID=$g timeout 900 python tools/span_log.py 60 2>&1 | grep -v "^ " | grep "^ovl \|^seq"
done
