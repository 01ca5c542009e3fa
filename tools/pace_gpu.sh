#!/bin/bash
# Paced victim-scan tickets + device intake: parity, kernel timeline, state microbench,
# full ncu captures of the intake kernels.  Output in gpurun_out/pace/.
O=gpurun_out/pace; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1; echo build rc=$?
timeout 1200 python -m pytest tests/test_gpu_parity.py -x -q -k "wide or sparse or reserve or dev_records or full_size_64k or c4_sweep or evict" > $O/pyt.log 2>&1; echo pyt rc=$?; tail -2 $O/pyt.log
timeout 300 python tools/vs_trace.py > $O/trace.json 2> $O/trace.err; echo trace rc=$?
timeout 600 python bench.py --state-only > $O/state.json 2> $O/state.err; echo state rc=$?
timeout 900 /usr/local/cuda/bin/ncu --set full --clock-control none --import-source on -k regex:'k_mark_acc|k_list' -c 2 \
  -o $O/prof_intake -f python bench.py --state-only > $O/ncu.log 2>&1; echo ncu rc=$?
