#!/bin/bash
# ncu --set full of every state kernel on bench.py's state microbench with 4 KiB blocks
# over 10.625 GiB of frames: the same block / frame counts as the bench (4.18 M / 2.78 M)
# on memory ncu's kernel replay can save and restore (it cannot back up 170 GiB).
# Launches: rep 0 (touch, discard, pressure) then rep 1.
O=gpurun_out/ncu; mkdir -p $O
timeout 1200 /usr/local/cuda/bin/ncu --set full --clock-control none --import-source on \
  -k regex:'k_classify|k_directive|k_victims' -c ${NCU_COUNT:-14} \
  -o $O/prof_state_${TAG:-x} -f python tools/state_bench.py 10.625 --block 4096 --reps 2 > $O/prof_state_${TAG:-x}.log 2>&1; echo "ncu rc=$?"
