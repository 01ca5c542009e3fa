#!/bin/bash
# per-launch device times of the state microbench (every kernel) + a full-set capture of
# the state kernels
O=gpurun_out/ncu; mkdir -p $O
timeout 600 /usr/local/cuda/bin/ncu --metrics gpu__time_duration.sum --clock-control none --csv \
  --log-file $O/state_launches.csv python tools/state_micro.py > $O/state_launches.log 2>&1; echo "launches rc=$?"
timeout 900 /usr/local/cuda/bin/ncu --set full --clock-control none --import-source on \
  -k regex:'k_classify|k_directive|k_victims' -c 12 -o $O/prof_state -f python tools/state_micro.py > $O/prof_state.log 2>&1; echo "ncu rc=$?"
