#!/bin/bash
# ncu evidence for a round (run under gpurun; one GPU).  Output in gpurun_out/ncu/.
O=gpurun_out/ncu; mkdir -p $O
NCU=/usr/local/cuda/bin/ncu
# (1) launch list of the bench command itself (metric-only pass, no replay)
timeout 900 $NCU --metrics gpu__time_duration.sum --clock-control none -k regex:'^k_' --csv \
  --log-file $O/launches_bench.csv python bench.py --steps 1 --warmup 1 --modes eager --no-e2e --no-cpu \
  --no-discard-bench > $O/bench_under_ncu.log 2>&1; echo "launches rc=$?"
# (2) full sets of the top kernel and the planning kernels on the small C3 run
timeout 900 $NCU --set full --clock-control none --import-source on -k regex:'k_service' -s 40 -c 3 \
  -o $O/prof_service -f python tools/profile_run.py eager > $O/prof_service.log 2>&1; echo "service rc=$?"
timeout 900 $NCU --set full --clock-control none --import-source on -k regex:'k_classify|k_victims|k_directive' -s 60 -c 6 \
  -o $O/prof_plan -f python tools/profile_run.py eager > $O/prof_plan.log 2>&1; echo "plan rc=$?"
ls -la $O
