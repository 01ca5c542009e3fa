#!/bin/bash
# one GPU round for state-kernel work: gpu parity tests, bench's state microbench, ncu of the state kernels
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
tail -3 gpurun_out/pytest_gpu.log
timeout 300 python tools/state_bench.py > gpurun_out/state_bench.json 2>&1
python - <<'PY'
import json
for l in open("gpurun_out/state_bench.json"):
    try:
        d = json.loads(l)
    except Exception:
        print(l[:300]); continue
    print({k: (round(v["ms"] * 1000, 2), round(v["frac"], 3)) for k, v in d.items() if isinstance(v, dict)})
PY
if [ -n "$TAG" ]; then bash tools/ncu_state_micro.sh; fi
