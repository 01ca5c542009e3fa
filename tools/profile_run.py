"""Small C3 run for ncu captures (kernel replay needs a modest memory footprint):
VGG-shaped Listing-6 trace, 2 MiB blocks, budget 8 GiB, 1.5x oversubscription, eager.

    ncu --set full -k regex:k_service -s 20 -c 2 -o gpurun_out/prof python tools/profile_run.py
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import tracegen as tg  # noqa: E402
from paper_conf_iiswc_zhucvhcr22_b200 import build, harness, um  # noqa: E402

mode = sys.argv[1] if len(sys.argv) > 1 else "eager"
budget = int(os.environ.get("PROF_BUDGET_GIB", "8")) << 30
t = tg.gen_c3(block_bytes=2 << 20, budget_bytes=budget, iterations=2)
build.build()
a = harness.make_arena(t, mode, flags=um.UM_F_APP_STAMP, host_pool_bytes=t.arena_bytes - t.budget_bytes + (1 << 30))
harness.alloc_buffers(a, t)
harness.issue(a, t, mode)
print(um.um_get_stats(a.handle))
a.close()
