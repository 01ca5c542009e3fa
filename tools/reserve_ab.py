"""A/B of proactive eviction (reading R12, um_config.reserve_blocks) on the bench's C3
step: eager iterations for each (reserve, schedule) pair on the same memory, CUDA events
on the paging stream.  Prints one JSON line per configuration.

    python tools/reserve_ab.py [--reserves 0,256,1024,4096] [--steps 3] [--warmup 2]
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import bench  # noqa: E402


def main():
    p = argparse.ArgumentParser()
    p.add_argument("--reserves", default="0,256,1024,4096")
    p.add_argument("--schedules", default="seq,overlap")
    p.add_argument("--steps", type=int, default=3)
    p.add_argument("--warmup", type=int, default=2)
    a = p.parse_args()
    sys.argv = [sys.argv[0]]
    args = bench.parse()
    import torch
    from paper_conf_iiswc_zhucvhcr22_b200 import build, um, harness
    build.build()
    dev = torch.device("cuda", 0)
    free, _ = torch.cuda.mem_get_info(dev)
    budget, arena_bytes, host_pool, clamp = bench.plan_sizes(args, free, 1)
    W, K = a.warmup, a.steps
    trace = bench.build_trace(args, budget, True, W + K)
    mem = um.Memory(args.block, arena_bytes, budget, host_pool_bytes=host_pool, device=0, threads=args.pin_threads)
    for sched in a.schedules.split(","):
        fl = um.UM_F_OVERLAP if sched == "overlap" else 0
        for r in [int(x) for x in a.reserves.split(",")]:
            try:
                res = bench.run_mode(torch, um, harness, mem, trace, "eager", W, K, flags_extra=fl, reserve=r)
            except um.UmError as e:   # e.g. the host-frame pool (arena - budget + 2 GiB) cannot hold the reserve
                print(json.dumps({"schedule": sched, "reserve_blocks": r, "error": str(e)}), flush=True)
                continue
            s = res["stats_per_iter"]
            print(json.dumps({"schedule": sched, "reserve_blocks": r, "reserve_gib": r * args.block / 2**30,
                              "iter_ms": res["iter_ms"], "iter_ms_each": res["iter_ms_each"],
                              "h2d_gb": s["h2d_bytes"] / 1e9, "d2h_gb": s["d2h_bytes"] / 1e9,
                              "evictions": s["evictions"], "plan_ms": res["timing"]["ms_plan"] / K,
                              "xfer_ms": res["timing"]["ms_xfer"] / K}), flush=True)


if __name__ == "__main__":
    main()
