#!/bin/bash
# Box facts, a default bench line and the state kernels' ncu capture.  Output in gpurun_out/final/.
O=gpurun_out/final; mkdir -p $O
(nvidia-smi topo -m; lscpu | head -20; numactl -H 2>/dev/null; free -g) > $O/box.txt 2>&1
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1; echo build rc=$?
s=$(date +%s); timeout 1500 python bench.py > $O/bench.json 2> $O/bench.err; echo "bench rc=$? wall=$(( $(date +%s) - s ))s"
python -c "import json;d=json.load(open('$O/bench.json'));print(d['iter_ms_each'], d['roofline']['frac'], d['clocks'])"
mkdir -p gpurun_out/ncu; bash tools/ncu_state.sh; cp -r gpurun_out/ncu $O/ 2>/dev/null
