#!/bin/bash
# bench line + launch list of the same command's kernels (ncu metric pass) for profiles/
mkdir -p gpurun_out/ncu
timeout 1200 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench rc=$?"
tail -2 gpurun_out/bench.err
timeout 1200 /usr/local/cuda/bin/ncu --metrics gpu__time_duration.sum --clock-control none -k regex:'^k_' --csv \
  --log-file gpurun_out/ncu/launches_bench.csv python bench.py --steps 1 --warmup 1 --modes eager --no-e2e --no-cpu \
  --no-discard-bench --no-compare > gpurun_out/ncu/bench_under_ncu.log 2>&1; echo "launches rc=$?"
