#!/bin/bash
# Step-0 probe of the GPU box.  Output under gpurun_out/probe/.
O=gpurun_out/probe; mkdir -p $O
( nvidia-smi -q > $O/nvidia_smi_q.txt; nvidia-smi topo -m > $O/topo.txt; lscpu > $O/lscpu.txt; nproc > $O/nproc.txt;
  numactl -H > $O/numa.txt 2>&1; free -g > $O/free.txt; cat /proc/meminfo > $O/meminfo.txt;
  nvidia-smi --query-gpu=index,pci.bus_id,clocks.sm,clocks.max.sm,memory.total,memory.used --format=csv > $O/gpu.csv;
  cat /sys/bus/pci/devices/*/current_link_speed 2>/dev/null | sort | uniq -c > $O/pcie_speeds.txt;
  nvidia-smi --query-gpu=pcie.link.gen.current,pcie.link.gen.max,pcie.link.width.current --format=csv > $O/pcie.csv ) 2>&1
timeout 300 ./tools/probe/probe bw > $O/bw.jsonl 2> $O/bw.err; echo "bw rc=$?"
timeout 300 ./tools/probe/probe pin ${PIN_CAP:-320} > $O/pin.jsonl 2> $O/pin.err; echo "pin rc=$?"
cat $O/bw.jsonl $O/pin.jsonl | head -100
