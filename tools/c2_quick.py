"""C2 streaming leg of bench.py alone (base / eager / lazy, closed-form check).

    python tools/c2_quick.py [pool_gib]
"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import bench  # noqa: E402
from paper_conf_iiswc_zhucvhcr22_b200 import build, harness, um  # noqa: E402

build.build()
GiB = 1 << 30
B = 2 << 20
pool = int(float(sys.argv[1] if len(sys.argv) > 1 else 40) * GiB)
budget = pool
mem = um.Memory(B, 2 * budget, budget, host_pool_bytes=pool, threads=8)
print(json.dumps(bench.c2_stream(torch, um, harness, mem, budget, pool)))
