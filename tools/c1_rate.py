"""bench.py's C1 small-op rate alone (ops/s through the API, and device-only us/op)."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import bench  # noqa: E402
from paper_conf_iiswc_zhucvhcr22_b200 import build, harness, um  # noqa: E402

build.build()
for _ in range(2):
    print(json.dumps(bench.c1_rate(torch, um, harness)))
