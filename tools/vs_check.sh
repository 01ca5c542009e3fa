#!/bin/bash
# Victim-scan check: kernel timeline (diagnostic build with -DUM_VS_TRACE), the parity
# tests that take the wide scan, and the state microbench.  Output in gpurun_out/vs/.
mkdir -p gpurun_out/vs
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/vs/build.log 2>&1; echo build rc=$?
timeout 300 python tools/vs_trace.py > gpurun_out/vs/trace.json 2> gpurun_out/vs/trace.err; echo trace rc=$?
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "wide or full_size_64k or c4_sweep or sparse or reserve" > gpurun_out/vs/pyt.log 2>&1; echo pyt rc=$?; tail -2 gpurun_out/vs/pyt.log
timeout 600 python bench.py --state-only > gpurun_out/vs/state.json 2> gpurun_out/vs/state.err; echo state rc=$?
