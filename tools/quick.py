"""Quick GPU checks of the small-op regime: C1 directives/s and the discard sweep
(functions from bench.py, without the 255 GiB C3 setup)."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import bench  # noqa: E402
from paper_conf_iiswc_zhucvhcr22_b200 import build, harness, um  # noqa: E402

build.build()
out = {"c1": bench.c1_rate(torch, um, harness)}
out["discard"] = [(r["bytes"], r["eager"]["kernel_us"], r["eager"]["api_us"], r["lazy"]["kernel_us"])
                  for r in bench.discard_bench(torch, um, reps=10)]
print(json.dumps(out))

out2 = bench.c4_sweep(torch, um, harness)
print(json.dumps(out2))
