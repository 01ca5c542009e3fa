"""The product's vectorised redundant-transfer report (paper_conf_iiswc_zhucvhcr22_b200/
rmt.py, used by bench.py on the CUDA path's transfer log) against the oracle's plain
rmt_analyze, on the oracle's transfer logs (CPU)."""
import numpy as np
import pytest

import tracegen as tg
from oracle.rmt import rmt_analyze, op_seq_starts
from oracle.sim import replay
from paper_conf_iiswc_zhucvhcr22_b200 import rmt as prmt


def _check(t, mode):
    log = replay(t, mode, record=True).log
    want = rmt_analyze(t, log)
    got = prmt.analyze(t, log)
    for k in ("h2d_bytes", "d2h_bytes", "rmt_h2d_bytes", "rmt_d2h_bytes", "rmt_bytes", "discarded_state_moves"):
        assert got[k] == want[k], (k, got[k], want[k])
    return got


@pytest.mark.parametrize("seed", range(30))
@pytest.mark.parametrize("mode", ["base", "eager", "lazy"])
def test_small_random(seed, mode):
    rng = np.random.default_rng(seed)
    nb, nf = int(rng.integers(2, 16)), int(rng.integers(1, 5))
    _check(tg.gen_small(seed, nblocks=nb, nframes=nf, n_ops=120, max_ranges=4, max_blocks=5), mode)


@pytest.mark.parametrize("mode", ["base", "eager", "lazy"])
def test_c1_c2_c3(mode):
    _check(tg.gen_c1(1).slice_ops(0, 3000), mode)
    _check(tg.gen_c2(16, 4, 3, block_bytes=4096), mode)
    for dead in (False, True):
        _check(tg.gen_c3(block_bytes=64 << 10, budget_bytes=192 << 20, iterations=2, workspace_bytes=4 << 20,
                         layers=tg.scale_layers(tg.VGG16, 1.0 / 512, 1.0 / 64), batch=8, discard_all_dead=dead), mode)


@pytest.mark.parametrize("seed", range(4))
def test_op_of_seq(seed):
    t = tg.gen_random(seed, block_bytes=4096, arena_bytes=256 * 4096, budget_bytes=20 * 4096, n_ops=300,
                      max_ranges=8, max_blocks=12, zipf_s=0.8)
    starts = op_seq_starts(t)
    seqs = np.arange(1, starts[-1] + 3)
    want = [max(i for i, s in enumerate(starts) if s <= q) for q in seqs]
    assert prmt.op_of_seq(t, seqs).tolist() == want
