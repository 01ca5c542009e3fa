"""N>1 path with the CUDA library (run on one B200): two ranks (gloo for the collective,
both on cuda:0 -- the driver's box has one GPU) each replay their own arena's trace through
libum with no exchange, then reduce the int64 counters and the max iteration time exactly
as bench.py does; the sums must equal the oracle's."""
import os
import socket

import pytest
import torch.multiprocessing as mp

pytestmark = pytest.mark.gpu


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, ws, port, q):
    import torch
    import torch.distributed as dist
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=ws)
    try:
        import tracegen as tg
        from oracle.sim import replay
        from paper_conf_iiswc_zhucvhcr22_b200 import harness, um
        from paper_conf_iiswc_zhucvhcr22_b200.dist import reduce_run, barrier
        torch.cuda.set_device(0)
        t = tg.gen_c1(200 + rank).slice_ops(0, 1500)      # per-rank trace, independent arenas
        barrier()
        g = harness.run_trace(t, "eager", flags=um.UM_F_APP_STAMP | um.UM_F_CHECK)
        red, tmax = reduce_run(g["stats"], 5.0 + rank)
        q.put((rank, replay(t, "eager").stats, g["stats"], red, tmax))
    finally:
        dist.destroy_process_group()


def test_two_ranks_libum_reduce():
    torch = pytest.importorskip("torch")
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    out = sorted(q.get(timeout=600) for _ in procs)
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    for rank, o, g, red, tmax in out:
        assert g == o, rank                      # each rank bit-exact with its oracle
        assert tmax == 6.0
    for k in out[0][1]:
        assert out[0][3][k] == out[0][1][k] + out[1][1][k]
