"""bench.py's state-kernel microbench alone (C3-64K tables over a 170 GiB frame budget;
2^21 random-block touch, 2^21-block discard), without the C3 run around it.

    python tools/state_bench.py [budget_gib]
"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import bench  # noqa: E402
from paper_conf_iiswc_zhucvhcr22_b200 import build, um  # noqa: E402

build.build()
GiB = 1 << 30
budget = int(float(sys.argv[1]) * GiB) if len(sys.argv) > 1 else 170 * GiB
budget = budget // (2 << 20) * (2 << 20)
arena = int(budget * 1.5) // (2 << 20) * (2 << 20)
mem = um.Memory(64 << 10, arena, budget, host_pool_bytes=1 << 30)
for rep in range(3):
    print(json.dumps(bench.state_bench(torch, um, mem, budget, arena, seed=rep)))
