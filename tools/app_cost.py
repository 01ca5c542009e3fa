"""How much of the C3 step the simulated application kernels take: the eager iteration
with and without UM_F_APP_STAMP, sequential and with UM_F_OVERLAP (R7), same memory.

    python tools/app_cost.py [iterations]
"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import bench  # noqa: E402
import tracegen as tg  # noqa: E402
from paper_conf_iiswc_zhucvhcr22_b200 import build, harness, um  # noqa: E402

build.build()
K = int(sys.argv[1]) if len(sys.argv) > 1 else 3
GiB = 1 << 30
free, _ = torch.cuda.mem_get_info(0)
B = 2 << 20
budget = min(170 * GiB, free - 5 * GiB) // B * B
trace = tg.gen_c3(block_bytes=B, budget_bytes=budget, oversub=1.5, iterations=K + 2, with_host_data=True)
mem = um.Memory(B, trace.arena_bytes, budget, host_pool_bytes=trace.arena_bytes - budget + 2 * GiB, threads=8)
out = {}
for name, fl in (("app_seq", um.UM_F_APP_STAMP), ("no_app", 0), ("app_overlap", um.UM_F_APP_STAMP | um.UM_F_OVERLAP)):
    # run_mode always ORs in UM_F_APP_STAMP; strip it for the no-app leg
    arena = harness.make_arena(trace, "eager", mem=mem, flags=fl | um.UM_F_TIMING)
    try:
        harness.alloc_buffers(arena, trace)
        bounds = harness.iteration_bounds(trace)
        ps = torch.cuda.ExternalStream(arena.stream_ptr)
        for i in range(2):
            harness.issue(arena, trace, "eager", *bounds[i])
        um.um_join(arena.handle)
        um.um_get_stats(arena.handle)
        um.um_timing(arena.handle, reset=True)
        evs = [torch.cuda.Event(enable_timing=True) for _ in range(K + 1)]
        evs[0].record(ps)
        for j in range(K):
            harness.issue(arena, trace, "eager", *bounds[2 + j])
            um.um_join(arena.handle)
            evs[j + 1].record(ps)
        evs[-1].synchronize()
        tm = um.um_timing(arena.handle, reset=True)
        out[name] = {"iter_ms": [evs[j].elapsed_time(evs[j + 1]) for j in range(K)],
                     "plan_ms": tm["ms_plan"] / K, "xfer_ms": tm["ms_xfer"] / K}
    finally:
        arena.close()
print(json.dumps(out))
