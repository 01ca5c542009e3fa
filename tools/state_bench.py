"""bench.py's state-kernel microbench alone (C3-64K tables over a 170 GiB frame budget;
2^21 random-block touch, 2^21-block discard, pressured 2^21 touch), without the C3 run.

    python tools/state_bench.py [budget_gib] [--block B]

--block 4096 with budget 10.625 GiB gives the same block and frame counts (4.18 M / 2.78 M)
on 11 GiB of frames, which ncu's kernel replay can save and restore.
"""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import bench  # noqa: E402
from paper_conf_iiswc_zhucvhcr22_b200 import build, um  # noqa: E402

p = argparse.ArgumentParser()
p.add_argument("budget_gib", nargs="?", type=float, default=170.0)
p.add_argument("--block", type=int, default=64 << 10)
p.add_argument("--reps", type=int, default=3)
a = p.parse_args()
build.build()
GiB = 1 << 30
budget = int(a.budget_gib * GiB) // (2 << 20) * (2 << 20)
arena = int(budget * 1.5) // (2 << 20) * (2 << 20)
mem = um.Memory(a.block, arena, budget, host_pool_bytes=1 << 30)
for rep in range(a.reps):
    print(json.dumps(bench.state_bench(torch, um, mem, budget, arena, seed=rep, block=a.block)))
