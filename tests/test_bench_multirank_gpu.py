"""bench.py's N>1 path end to end on the one-GPU box: torchrun with 2 ranks sharing cuda:0
(BENCH_SHARE_GPU=1: gloo collectives), small budget; rank 0 prints one line whose value
and counters are the whole job's."""
import json
import os
import socket
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def test_two_rank_bench_line():
    torch = pytest.importorskip("torch")
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    env = dict(os.environ, BENCH_SHARE_GPU="1")
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "2", "--master-addr",
           "127.0.0.1", "--master-port", str(_port()), os.path.join(ROOT, "bench.py"), "--gpus", "2", "--steps", "2",
           "--warmup", "3", "--budget-gib", "8", "--no-compare", "--no-discard-bench", "--no-state-bench",
           "--no-cpu"]
    out = subprocess.run(cmd, capture_output=True, text=True, timeout=900, cwd=ROOT, env=env)
    assert out.returncode == 0, out.stderr[-3000:]
    lines = [x for x in out.stdout.splitlines() if x.startswith("{")]
    assert len(lines) == 1                      # rank 0 only
    d = json.loads(lines[0])
    assert d["n_gpus"] == 2 and d["scaling"] == "weak"
    assert d["value"] == pytest.approx(2 / (d["ms_per_step"] / 1e3), rel=1e-6)
    per_rank = d["stats_per_iter"]["eager"]
    tot = d["stats_all_ranks"]["counters"]
    # identical traces on both ranks: the all-reduced counters are twice one rank's
    assert tot["h2d_bytes"] == 2 * 2 * per_rank["h2d_bytes"] and tot["ops"] == 2 * 2 * per_rank["ops"]
