"""Per-span timing of one C3 iteration (UM_F_TIMING spans with UM_SPAN_LOG), sequential
app kernels vs UM_F_OVERLAP, to find where planning time goes.

    python tools/span_log.py [budget_gib]
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
budget = int(float(sys.argv[1] if len(sys.argv) > 1 else 60) * GiB) // B * B


class A:
    block, oversub, budget_gib = B, 1.5, budget / GiB
    discard_all_dead = False


trace = bench.build_trace(A, budget, True, 3)
arena_bytes = trace.arena_bytes
mem = um.Memory(B, arena_bytes, budget, host_pool_bytes=arena_bytes - budget + 2 * GiB, threads=8)
os.makedirs("gpurun_out", exist_ok=True)
variants = [("seq", 0, um.UM_F_APP_STAMP, {}), ("ovl", um.UM_F_OVERLAP, um.UM_F_APP_STAMP, {})]
if os.environ.get("SPAN_ALL"):
    variants += [("ovl_noapp", um.UM_F_OVERLAP, 0, {}),
                 ("ovl_serial", um.UM_F_OVERLAP, um.UM_F_APP_STAMP, {"UM_OVERLAP_SERIAL": "1"})]
for tag, fl, app, env in variants:
    os.environ.update(env)
    path = f"gpurun_out/spans_{tag}.txt"
    if os.path.exists(path):
        os.remove(path)
    arena = harness.make_arena(trace, "eager", mem=mem, flags=app | um.UM_F_TIMING | fl)
    harness.alloc_buffers(arena, trace)
    bounds = harness.iteration_bounds(trace)
    for i in range(2):
        harness.issue(arena, trace, "eager", *bounds[i])
    um.um_get_stats(arena.handle)
    um.um_timing(arena.handle, reset=True)
    os.environ["UM_SPAN_LOG"] = path
    ps = torch.cuda.ExternalStream(arena.stream_ptr)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(ps)
    harness.issue(arena, trace, "eager", *bounds[2])
    um.um_join(arena.handle)
    e1.record(ps)
    e1.synchronize()
    t = um.um_timing(arena.handle, reset=True)
    t["iter_ms"] = e0.elapsed_time(e1)
    del os.environ["UM_SPAN_LOG"]
    arena.close()
    for k in env:
        del os.environ[k]
    rows = [l.split() for l in open(path)]
    plan = sorted(((float(r[2]), int(r[0])) for r in rows if r[1] == "0"), reverse=True)
    print(tag, json.dumps(t))
    ops = trace.ops.tolist()
    for ms, sq in plan[:12]:
        print(f"  {ms:8.3f} ms  seq {sq}  op {ops[sq - 1] if sq - 1 < len(ops) else None}")
    print("  plan total", sum(p[0] for p in plan), "n", len(plan))
