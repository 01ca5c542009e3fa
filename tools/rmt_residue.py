"""Diagnostic: time the RMT leg's eager iteration before and after the state microbench
(is there a residue of the state leg on later C3 iterations?).  One JSON line per phase."""
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import bench  # noqa: E402


def main():
    sys.argv = [sys.argv[0]]
    args = bench.parse()
    import torch
    from paper_conf_iiswc_zhucvhcr22_b200 import build, um, harness
    build.build()
    free, _ = torch.cuda.mem_get_info(0)
    budget, arena_bytes, host_pool, _ = bench.plan_sizes(args, free, 1)
    trace = bench.build_trace(args, budget, True, 4)
    mem = um.Memory(args.block, arena_bytes, budget, host_pool_bytes=host_pool, device=0, threads=args.pin_threads)

    def c3(tag):
        r = bench.run_mode(torch, um, harness, mem, trace, "eager", 2, 2)
        print(json.dumps({"phase": tag, "iter_ms_each": r["iter_ms_each"]}), flush=True)

    def rmt(tag):
        t0 = time.time()
        r = bench.rmt_leg(torch, um, harness, mem, budget, args.oversub, args.block)
        print(json.dumps({"phase": tag, "listing6": r["listing6_literal"]["iter_ms"],
                          "all_dead": r["discard_all_dead"]["iter_ms"], "wall_s": time.time() - t0}), flush=True)
    c3("c3 first")
    rmt("rmt before state")
    bench.state_runs(torch, um, mem, budget, arena_bytes)
    c3("c3 after state")
    rmt("rmt after state")


if __name__ == "__main__":
    main()
