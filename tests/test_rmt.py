"""Pins of oracle/rmt.py (redundant-transfer accounting, DESIGN R8)
against things other than itself: Fig. 2's two RMTs (hand-enumerated), the C2 closed
form, and a second formulation (a forward, versioned flat memory) on brute-forced
traces."""
import itertools

import numpy as np
import pytest

import tracegen as tg
from oracle.rmt import rmt_analyze, rmt_compare, log_by_op, op_seq_starts, H2D, D2H
from oracle.sim import replay, G, H

B = 4096


def _e1(with_discard=True):
    tb = tg.TraceBuilder(B, 2 * B, B)
    tb.touch([(0, B, tg.ACC_WRITE)])
    if with_discard:
        tb.discard(0, B, lazy_ok=True)
    tb.touch([(B, B, tg.ACC_WRITE)])
    tb.touch([(0, B, tg.ACC_WRITE)])
    return tb.build()


def _log(trace, mode):
    o = replay(trace, mode, record=True)
    return o.log


def test_e1_fig2_hand_log():
    """Fig. 2 (L112, L131): with discard off, the eviction of A (3) and its migration back
    (4) are the redundant transfers; the write-back of B is required (B is read at the end)."""
    t = _e1()
    # ops: 0 touch A(W); 1 discard A; 2 touch B(W); 3 touch A(W) -- one frame
    hand = [(2, D2H, 0, G), (3, D2H, 1, G), (3, H2D, 0, H)]
    r = rmt_analyze(t, hand, by_op=True)
    assert r["rmt_d2h_bytes"] == B and r["rmt_h2d_bytes"] == B and r["rmt_bytes"] == 2 * B
    assert r["reasons"]["dead"] == 2 * B                 # both moved A after its discard
    assert r["discarded_state_moves"] == 0
    # the oracle's own logs, mapped to ops, are exactly these transfers
    base = [x for x in log_by_op(t, _log(t, "base")) if x[1] != "ZF"]
    assert sorted(base) == sorted(hand)
    eager = [x for x in log_by_op(t, _log(t, "eager")) if x[1] != "ZF"]
    assert eager == [(3, D2H, 1, G)]
    c = rmt_compare(rmt_analyze(t, _log(t, "base")), rmt_analyze(t, _log(t, "eager")))
    assert c == {"rmt_base_bytes": 2 * B, "rmt_left_bytes": 0, "avoided_bytes": 2 * B, "discarded_state_moves": 0}


def test_e1_without_discard_still_redundant_by_overwrite():
    """L34: A is overwritten before being read, so its eviction and migration are
    redundant even when the program never discards it (reason: overwritten)."""
    t = _e1(with_discard=False)
    hand = [(1, D2H, 0, G), (2, D2H, 1, G), (2, H2D, 0, H)]
    r = rmt_analyze(t, hand, by_op=True)
    assert r["rmt_bytes"] == 2 * B and r["reasons"]["overwritten"] == 2 * B


def test_read_makes_transfer_required():
    tb = tg.TraceBuilder(B, 2 * B, B)
    tb.touch([(0, B, tg.ACC_WRITE)])
    tb.touch([(B, B, tg.ACC_WRITE)])
    tb.touch([(0, B, tg.ACC_READ | tg.ACC_WRITE)])
    t = tb.build()
    r = rmt_analyze(t, _log(t, "eager"))
    assert r["d2h_bytes"] == 2 * B and r["h2d_bytes"] == B and r["rmt_bytes"] == 0


@pytest.mark.parametrize("F,c,P", [(8, 2, 3), (16, 4, 4), (64, 8, 2), (6, 3, 2)])
def test_c2_closed_form(F, c, P):
    """in base mode every transfer of the FIR-like stream is
    redundant, RMT_base = (4P-3)F blocks; with discard nothing moves, RMT_left = 0."""
    t = tg.gen_c2(F, c, P, block_bytes=B)
    rb = rmt_analyze(t, _log(t, "base"))
    assert rb["rmt_bytes"] == (4 * P - 3) * F * B == rb["h2d_bytes"] + rb["d2h_bytes"]
    for mode in ("eager", "lazy"):
        rd = rmt_analyze(t, _log(t, mode))
        assert rd["rmt_bytes"] == 0 and rd["h2d_bytes"] == rd["d2h_bytes"] == 0


def _seq_starts_by_replay(trace):
    starts = []
    o = replay(trace, "base", stop=0)
    from oracle.sim import apply_op
    for op in trace.iter_ops():
        starts.append(o.clock + 1)
        apply_op(o, op, "base")
    return starts


@pytest.mark.parametrize("seed", range(6))
def test_op_seq_starts_matches_the_oracle_numbering(seed):
    t = tg.gen_small(seed, nblocks=12, nframes=3, n_ops=200, max_ranges=4, max_blocks=6)
    assert op_seq_starts(t) == _seq_starts_by_replay(t)


def _versioned_redundant(trace, recs):
    """Second formulation: replay the data events on a flat memory whose cells hold a
    version (a fresh id per write, None once discarded); a transfer at op t moves the
    version current before op t's events; it is required iff that version is not None
    and is read at op t or later (or is the final content)."""
    Bk = trace.block_bytes
    ops = list(trace.iter_ops())
    ver, nxt = {}, itertools.count(1)
    moved = {}                          # transfer index -> version moved
    reads_of = {}                       # version -> last op that reads it (final contents: len(ops))
    by_t = {}
    for i, (t, k, b, p) in enumerate(recs):
        by_t.setdefault(t, []).append((i, b))
    for t, (kind, flags, off, ln, accs) in enumerate(ops):
        for (i, b) in by_t.get(t, ()):
            moved[i] = ver.get(b, ("init", b))
        if kind == 0:
            rd, wr = set(), set()
            for (o, n, kk) in accs:
                r = range(o // Bk, (o + n - 1) // Bk + 1) if n else range(0)
                if kk & tg.ACC_READ:
                    rd.update(r)
                if kk & tg.ACC_WRITE:
                    wr.update(r)
            for b in rd:                # the application reads, then writes
                v = ver.get(b, ("init", b))
                if v is not None:
                    reads_of[v] = t
            for b in wr:
                ver[b] = ("w", next(nxt))
        elif kind in (2, 5):            # discard, free
            lo = -(-off // Bk)
            for b in range(lo, max(lo, (off + ln) // Bk)):
                ver[b] = None
        elif kind == 4:
            for b in range(off // Bk, (off + ln - 1) // Bk + 1) if ln else ():
                ver[b] = ("w", next(nxt))
    for b in range(trace.arena_bytes // Bk):
        v = ver.get(b, ("init", b))
        if v is not None:
            reads_of[v] = len(ops)      # final contents are checked
    red = 0
    for i, (t, k, b, p) in enumerate(recs):
        if k in (H2D, D2H):
            v = moved[i]
            if v is None or reads_of.get(v, -1) < t:
                red += Bk
    return red


@pytest.mark.parametrize("seed", range(40))
@pytest.mark.parametrize("mode", ["base", "eager", "lazy"])
def test_second_formulation(seed, mode):
    rng = np.random.default_rng(seed)
    nb, nf = int(rng.integers(2, 10)), int(rng.integers(1, 4))
    t = tg.gen_small(seed, nblocks=nb, nframes=nf, n_ops=60, max_ranges=3, max_blocks=4)
    recs = log_by_op(t, _log(t, mode))
    r = rmt_analyze(t, recs, by_op=True)
    # ("init", b) = the zero-initialised content of a never-written block
    assert r["rmt_bytes"] == _versioned_redundant(t, recs)
    if mode != "base":
        assert r["discarded_state_moves"] == 0


def _partial_tail_blocks(t):
    """Blocks that some discard covers only partly and no discard covers fully (A4,
    §5.4: the discard ignores them)."""
    Bk = t.block_bytes
    part, full = set(), set()
    for kind, flags, off, ln, accs in t.iter_ops():
        if kind == 2 and ln:
            part.update(range(off // Bk, (off + ln - 1) // Bk + 1))
            lo = -(-off // Bk)
            full.update(range(lo, max(lo, (off + ln) // Bk)))
    return part - full


def test_c3_small_rmt_left():
    """Listing 6 never discards output_1 or data (SURVEY §8(d) literal gap); the
    --discard-all-dead variant discards them after backward_1, and then the only
    redundant transfers left in discard mode are of buffer tails that a discard covers
    only partly (the discard ignores partial blocks, A4 / §5.4; NEXT-1's page
    masks are the remedy)."""
    kw = dict(block_bytes=64 << 10, budget_bytes=192 << 20, iterations=2, workspace_bytes=4 << 20,
              layers=tg.scale_layers(tg.VGG16, 1.0 / 512, 1.0 / 64), batch=8)
    res = {}
    for dead in (False, True):
        t = tg.gen_c3(discard_all_dead=dead, **kw)
        rb = rmt_analyze(t, _log(t, "base"))
        for mode in ("eager", "lazy"):
            rd = rmt_analyze(t, _log(t, mode))
            c = rmt_compare(rb, rd)
            assert c["discarded_state_moves"] == 0
            assert c["rmt_base_bytes"] > 0
            assert c["rmt_left_bytes"] <= c["rmt_base_bytes"]
            res[(dead, mode)] = c
        if dead:
            tails = _partial_tail_blocks(t)
            for mode in ("eager", "lazy"):
                left = rmt_analyze(t, _log(t, mode), detail=True)["records"]
                assert left and all(b in tails for (_t, _k, b, _r) in left)
    assert res[(False, "eager")]["rmt_left_bytes"] > res[(True, "eager")]["rmt_left_bytes"]
