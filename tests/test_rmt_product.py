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


@pytest.mark.parametrize("mode", ["base", "eager", "lazy"])
def test_two_level_logs(mode):
    """Per-page logs of the two-level oracle (oracle/chunks.py, NEXT-1)."""
    from oracle.chunks import replay_chunks
    P = 64 << 10
    t = tg.gen_c3(block_bytes=2 << 20, budget_bytes=384 << 20, iterations=2, workspace_bytes=5 << 20,
                  layers=tg.scale_layers(tg.VGG16, 1.0 / 64, 1.0 / 16), batch=6, discard_all_dead=True)
    log = replay_chunks(t, P, mode, record=True).log
    want = rmt_analyze(t, log, page_bytes=P)
    got = prmt.analyze(t, log, page_bytes=P)
    for k in ("h2d_bytes", "d2h_bytes", "rmt_h2d_bytes", "rmt_d2h_bytes", "rmt_bytes", "discarded_state_moves"):
        assert got[k] == want[k], (k, got[k], want[k])
    if mode != "base":
        # what is left is only pages that a discard covers in part (A4 at page level),
        # far less than the single-level run leaves (whole-chunk tails)
        from oracle.sim import replay
        single = rmt_analyze(t, replay(t, mode, record=True).log)
        left = rmt_analyze(t, log, page_bytes=P, detail=True)["records"]
        part, full = set(), set()
        for kind, flags, off, ln, accs in t.iter_ops():
            if kind == 2 and ln:
                part.update(range(off // P, (off + ln - 1) // P + 1))
                full.update(range(-(-off // P), (off + ln) // P))
        assert all(q in part - full for (_t, _k, q, _r) in left)
        assert got["rmt_bytes"] < single["rmt_bytes"]
