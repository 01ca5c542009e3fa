#!/bin/bash
# ncu --set full of the victim kernels (k_victims_scan / k_victims_apply) of the
# pressured touch in tools/state_micro.py.  Output in gpurun_out/vs/.
O=gpurun_out/vs; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 900 /usr/local/cuda/bin/ncu --set full --clock-control none --import-source on \
  -k regex:'k_victims' -c 2 -o $O/prof_vict -f python tools/state_micro.py > $O/prof_vict.log 2>&1; echo "full rc=$?"
