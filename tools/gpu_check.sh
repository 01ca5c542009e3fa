#!/bin/bash
# One GPU pass: build, parity suite, smoke, a short bench line.  Logs under gpurun_out/.
O=gpurun_out; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1; echo "build rc=$?"
s=$(date +%s)
timeout ${PYT_TIMEOUT:-1500} python -m pytest tests -m gpu -x -q ${PYT_ARGS:-} > $O/pytest_gpu.log 2>&1; echo "pytest rc=$? wall=$(( $(date +%s) - s ))s"
tail -3 $O/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?"; tail -1 $O/smoke.log
if [ -n "$BENCH_ARGS" ]; then
  s=$(date +%s)
  timeout ${BENCH_TIMEOUT:-1800} python bench.py $BENCH_ARGS > $O/bench.json 2> $O/bench.err; echo "bench rc=$? wall=$(( $(date +%s) - s ))s"
  tail -2 $O/bench.err; head -c 600 $O/bench.json
fi
