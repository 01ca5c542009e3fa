#!/bin/bash
# ncu --set full of the state kernels on bench.py's state microbench (tools/state_bench.py)
O=gpurun_out/ncu; mkdir -p $O
timeout 300 python tools/state_bench.py > $O/state_bench.json 2>&1; echo "state_bench rc=$?"; head -c 3000 $O/state_bench.json; echo
timeout 1200 /usr/local/cuda/bin/ncu --set full --clock-control none --import-source on \
  -k regex:'k_classify|k_directive|k_victims' -c ${NCU_COUNT:-7} \
  -o $O/prof_state_full -f python tools/state_bench.py > $O/prof_state_full.log 2>&1; echo "ncu rc=$?"
