#!/bin/bash
# ncu evidence for a round (run under gpurun; one GPU).  Output in gpurun_out/ncu/.
#  (1) launch list of the bench command (eager step only; metric-only pass)
#  (2) per-launch DRAM and PCIe bytes of k_service in the bench configuration
#  (3) one --set full capture of a k_service launch of the bench configuration
O=gpurun_out/ncu; mkdir -p $O
NCU=/usr/local/cuda/bin/ncu
BENCH="python bench.py --steps 1 --warmup 3 --modes eager --no-e2e --no-cpu --no-discard-bench --no-compare --no-state-bench"
timeout 1500 $NCU --metrics gpu__time_duration.sum --clock-control none -k regex:'^k_' --csv \
  --log-file $O/launches_bench.csv $BENCH > $O/bench_under_ncu.log 2>&1; echo "launches rc=$?"
timeout 1500 $NCU --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,pcie__read_bytes.sum,pcie__write_bytes.sum \
  --clock-control none -k regex:'k_service' -s 170 -c 60 --csv --log-file $O/service_traffic.csv $BENCH > $O/traffic.log 2>&1; echo "traffic rc=$?"
timeout 1500 $NCU --set full --clock-control none --import-source on -k regex:'k_service' -s 200 -c 1 \
  -o $O/prof_service -f $BENCH > $O/prof_service.log 2>&1; echo "full rc=$?"
ls -la $O
