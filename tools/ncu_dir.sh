#!/bin/bash
O=gpurun_out/ncu; mkdir -p $O
timeout 600 /usr/local/cuda/bin/ncu --set full --clock-control none --import-source on -k regex:'k_directive|k_classify' -c 3 \
  -o $O/prof_dir -f python tools/state_micro.py > $O/prof_dir.log 2>&1; echo "ncu rc=$?"
