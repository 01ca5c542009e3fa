"""world_size-2 gloo tests of the N>1 path (CPU): each rank replays its own arena's trace
(independent units, no exchange) and only the final counters/time are reduced."""
import os
import socket

import pytest
import torch.multiprocessing as mp


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, ws, port, q):
    import torch.distributed as dist
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=ws)
    try:
        import tracegen as tg
        from oracle.sim import replay
        from paper_conf_iiswc_zhucvhcr22_b200.dist import reduce_run, world
        assert world() == (rank, ws)
        # independent per-rank arenas: per-rank seed, no exchange during the replay
        t = tg.gen_c1(100 + rank).slice_ops(0, 1500)
        s = dict(replay(t, "eager").stats)
        s["big"] = (1 << 60) + 2 * rank + 1          # beyond 2^53: the reduce must be int64-exact
        red, tmax = reduce_run(s, 10.0 + rank)
        q.put((rank, s, red, tmax))
    finally:
        dist.destroy_process_group()


def test_gloo_ws2_reduce_counters_and_max_time():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    out = [q.get(timeout=120) for _ in procs]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    out.sort()
    s0, s1 = out[0][1], out[1][1]
    for rank, s, red, tmax in out:
        assert tmax == 11.0
        for k in s0:
            assert red[k] == s0[k] + s1[k]
        assert red["big"] == (1 << 61) + 4


def test_reduce_run_single_process_is_identity():
    from paper_conf_iiswc_zhucvhcr22_b200.dist import reduce_run
    s, t = reduce_run({"a": 3, "b": 4}, 5.0)
    assert s == {"a": 3, "b": 4} and t == 5.0
