#!/bin/bash
O=gpurun_out/ncu; mkdir -p $O
timeout 300 python tools/state_micro.py > $O/state_micro.json 2>&1; echo "micro rc=$?"; cat $O/state_micro.json | head -c 3000; echo
timeout 900 /usr/local/cuda/bin/ncu --set full --clock-control none --import-source on -k regex:'k_classify|k_directive|k_victims' -c 6 \
  -o $O/prof_state -f python tools/state_micro.py > $O/prof_state.log 2>&1; echo "ncu rc=$?"
