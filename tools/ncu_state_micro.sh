#!/bin/bash
# ncu --set full of every state kernel on tools/state_micro.py (12 GiB of frames: ncu's
# device-memory save/restore of kernel replay cannot back up the 170 GiB bench arena)
O=gpurun_out/ncu; mkdir -p $O
timeout 1200 /usr/local/cuda/bin/ncu --set full --clock-control none --import-source on \
  -k regex:'k_classify|k_directive|k_victims' -c ${NCU_COUNT:-12} \
  -o $O/prof_state_${TAG:-x} -f python tools/state_micro.py > $O/prof_state_${TAG:-x}.log 2>&1; echo "ncu rc=$?"
