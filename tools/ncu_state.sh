#!/bin/bash
# --set full of the state kernels on the 2^21-block microbench with 4 KiB blocks
# (tools/state_micro.py: same tables as the bench's C3-64K microbench, 12 GiB of frames,
# so kernel replay can back up the memory).  Output in gpurun_out/ncu/.
O=gpurun_out/ncu; mkdir -p $O
timeout 1200 /usr/local/cuda/bin/ncu --set full --clock-control none --import-source on \
  -k regex:'k_classify|k_directive|k_victims' -c 6 -o $O/prof_state -f python tools/state_micro.py \
  > $O/prof_state.log 2>&1; echo "state full rc=$?"
