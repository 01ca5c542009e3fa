#!/bin/bash
# Device-resident records (um_touch_batch_dev): parity tests, the state microbench and a
# launch list of the intake kernels.
O=gpurun_out/devrec; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1; echo build rc=$?
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "dev_records or state_micro" > $O/pyt.log 2>&1; echo pyt rc=$?; tail -3 $O/pyt.log
timeout 600 python bench.py --state-only > $O/state.json 2> $O/state.err; echo state rc=$?; tail -3 $O/state.err
timeout 900 /usr/local/cuda/bin/ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none \
  -k regex:'k_mark_acc|k_list|k_classify' -c 12 --csv --log-file $O/launches.csv python bench.py --state-only > $O/ncu.log 2>&1; echo ncu rc=$?
