#!/bin/bash
O=gpurun_out/mark; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 900 /usr/local/cuda/bin/ncu --set full --clock-control none --import-source on -k regex:'k_mark_acc|k_list' -c 2 \
  -o $O/prof -f python bench.py --state-only > $O/ncu.log 2>&1; echo ncu rc=$?
