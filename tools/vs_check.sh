mkdir -p gpurun_out/vs
timeout 300 python tools/vs_trace.py > gpurun_out/vs/trace.json 2> gpurun_out/vs/trace.err; echo trace rc=$?
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "wide_victim or full_size_64k or c4_sweep or device_intake_wide" > gpurun_out/vs/pyt.log 2>&1; echo pyt rc=$?; tail -2 gpurun_out/vs/pyt.log
timeout 600 python bench.py --state-only > gpurun_out/vs/state.json 2> gpurun_out/vs/state.err; echo state rc=$?
