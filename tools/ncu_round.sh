#!/bin/bash
# ncu evidence for a round (run under gpurun; one GPU).  Output in gpurun_out/ncu/.
#  (1) launch list of the bench command (eager step only; metric-only pass)
#  (2) DRAM and PCIe bytes of every k_service launch of the bench's timed iteration
#      (W = 3 warm-up iterations x 167 launches skipped; single-pass metrics, no replay)
#  (3) one --set full capture of a k_service launch of a small C3 run (tools/profile_run.py;
#      kernel replay of the bench-sized run would back up 260 GB of memory)
O=gpurun_out/ncu; mkdir -p $O
NCU=/usr/local/cuda/bin/ncu
BENCH="python bench.py --steps 1 --warmup 3 --modes eager --no-e2e --no-cpu --no-discard-bench --no-compare --no-state-bench"
timeout 1500 $NCU --metrics gpu__time_duration.sum --clock-control none -k regex:'^k_' --csv \
  --log-file $O/launches_bench.csv $BENCH > $O/bench_under_ncu.log 2>&1; echo "launches rc=$?"
timeout 1500 $NCU --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,pcie__read_bytes.sum,pcie__write_bytes.sum \
  --clock-control none -k regex:'k_service' -s 501 -c 167 --csv --log-file $O/service_traffic.csv $BENCH > $O/traffic.log 2>&1; echo "traffic rc=$?"
timeout 900 $NCU --set full --clock-control none --import-source on -k regex:'k_service' -s 40 -c 2 \
  -o $O/prof_service -f python tools/profile_run.py eager > $O/prof_service.log 2>&1; echo "full rc=$?"
ls -la $O
