#!/bin/bash
# Re-check: the state-microbench parity tests (medium, full size) and a short base/eager C3 bench.
O=gpurun_out/recheck; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1; echo build rc=$?
timeout 1200 python -m pytest tests/test_gpu_parity.py -x -q -k "state_micro" > $O/pyt.log 2>&1; echo pyt rc=$?; tail -3 $O/pyt.log
timeout 900 python bench.py --steps 4 --warmup 2 --modes base,eager --no-compare --no-state-bench --no-discard-bench --no-e2e --no-cpu > $O/bench.json 2> $O/bench.err; echo bench rc=$?
python -c "import json;d=json.load(open('$O/bench.json'));print(d['iter_ms_each'], d['link_peak'], d['clocks'])"
