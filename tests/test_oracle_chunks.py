"""Pins of the two-level oracle (oracle/chunks.py), CPU only:
hand-derived scenarios, the reduction to the single-level oracle when no discard is
partial, and page-level invariants."""
import numpy as np
from hypothesis import HealthCheck, given, settings
from hypothesis import strategies as hst

import tracegen as tg
from oracle.chunks import replay_chunks
from oracle.sim import ST_NAMES, replay

P = 4096            # page
PPC = 4             # pages per chunk in the scenarios
C = P * PPC         # chunk


def _s(seq, q):
    return (seq << 32) | q


def _trace(nchunks, nframes, ops):
    tb = tg.TraceBuilder(C, nchunks * C, nframes * C)
    for op in ops:
        kind = op[0]
        if kind == "touch":      # ("touch", [(first page, n pages, "R"|"W")...])
            tb.touch([(q * P, n * P, tg.ACC_WRITE if k == "W" else tg.ACC_READ) for q, n, k in op[1]])
        elif kind == "discard":  # ("discard", first page, n pages, lazy)
            tb.discard(op[1] * P, op[2] * P, lazy_ok=op[3])
        elif kind == "discard_bytes":
            tb.discard(op[1], op[2])
        elif kind == "prefetch":
            tb.prefetch(op[1] * P, op[2] * P, op[3])
        elif kind == "evict":
            tb.evict(op[1] * C)
        elif kind == "host_write":
            tb.host_write(op[1] * P, op[2] * P)
    return tb.build()


# ------------------------------------------------------------------ hand-derived scenarios
def test_partial_discard_skips_dead_pages_both_ways():
    """Chunks A (pages 0-3), B (4-7), one frame.  s1 touch A:W (ZF 4 pages); s2 discard
    pages 0-1 (dead 0b0011, A stays G in USED: no split, L211); s3 touch B:W evicts A:
    D2H of pages 2-3 only, pages 0-1 avoided (L196-198); s4 touch A:R evicts B (4 pages
    D2H) and migrates A: pages 2-3 H2D, pages 0-1 zero-filled (L200); the touch revives
    them.  Contents: A = 0, 0, s1, s1; B = s3 on the host."""
    t = _trace(2, 1, [("touch", [(0, 4, "W")]), ("discard", 0, 2, False), ("touch", [(4, 4, "W")]),
                      ("touch", [(0, 4, "R")])])
    o = replay_chunks(t, P, "eager")
    o.check_conservation()
    s = o.stats
    assert (s["zf_bytes"], s["d2h_bytes"], s["h2d_bytes"]) == (10 * P, 6 * P, 2 * P)
    assert (s["d2h_avoided_bytes"], s["h2d_avoided_bytes"]) == (2 * P, 2 * P)
    assert (s["evictions"], s["faults"], s["unmaps"]) == (2, 3, 0)
    assert [ST_NAMES[x] for x in o.st] == ["G", "H"]
    assert o.dead == [0, 0]
    assert o.contents() == [0, 0, _s(1, 2), _s(1, 3)] + [_s(3, q) for q in range(4, 8)]
    b = replay_chunks(t, P, "base").stats      # discard off: whole chunks move
    assert (b["zf_bytes"], b["d2h_bytes"], b["h2d_bytes"]) == (8 * P, 8 * P, 4 * P)


def test_lazy_partial_discard_needs_prefetch():
    """s1 touch A:W; s2 discard_lazy pages 0-1 (dead = lazy = 0b0011); s3 touch page 0:W
    is a hit and does not revive a lazy page (A8); s4 touch B:W evicts A writing back
    pages 2-3 only, so s3's write to page 0 is lost (defined, A8); s5 prefetch A to the
    GPU evicts B, zero-fills pages 0-1, migrates 2-3 and revalidates all pages (A17)."""
    t = _trace(2, 1, [("touch", [(0, 4, "W")]), ("discard", 0, 2, True), ("touch", [(0, 1, "W")]),
                      ("touch", [(4, 4, "W")]), ("prefetch", 0, 4, tg.DST_GPU)])
    o = replay_chunks(t, P, "lazy")
    o.check_conservation()
    s = o.stats
    assert (s["zf_bytes"], s["d2h_bytes"], s["h2d_bytes"]) == (10 * P, 6 * P, 2 * P)
    assert (s["d2h_avoided_bytes"], s["h2d_avoided_bytes"]) == (2 * P, 2 * P)
    assert (s["hits"], s["faults"], s["evictions"]) == (1, 2, 2)
    assert o.dead == [0, 0] and o.lazy == [0, 0]
    assert o.contents() == [0, 0, _s(1, 2), _s(1, 3)] + [_s(4, q) for q in range(4, 8)]


def test_partial_discard_of_host_resident_chunk():
    """s1 touch A:W; s2 touch B:W evicts A whole (4 pages D2H); s3 discard pages 2-3 of
    the host-resident A (its host copy of them is released, R1); s4 touch A:R evicts B and
    migrates only pages 0-1, zero-filling 2-3 (h2d_avoided 2 pages)."""
    t = _trace(2, 1, [("touch", [(0, 4, "W")]), ("touch", [(4, 4, "W")]), ("discard", 2, 2, False),
                      ("touch", [(0, 4, "R")])])
    o = replay_chunks(t, P, "eager")
    o.check_conservation()
    s = o.stats
    assert (s["zf_bytes"], s["d2h_bytes"], s["h2d_bytes"]) == (10 * P, 8 * P, 2 * P)
    assert (s["d2h_avoided_bytes"], s["h2d_avoided_bytes"]) == (0, 2 * P)
    assert o.contents() == [_s(1, 0), _s(1, 1), 0, 0] + [_s(2, q) for q in range(4, 8)]


def test_unaligned_discard_marks_fully_covered_pages_only():
    """A discard of [P/2, P/2 + 2P) covers page 1 fully and pages 0 and 2 in part (A4 at
    page granularity): only page 1 is dead."""
    t = _trace(2, 2, [("touch", [(0, 4, "W")]), ("discard_bytes", P // 2, 2 * P)])
    o = replay_chunks(t, P, "eager")
    assert o.dead == [0b0010, 0]
    assert [ST_NAMES[x] for x in o.st] == ["G", "U"]


def test_whole_chunk_discard_is_chunk_level():
    """A discard covering chunk A entirely and B in part: A goes to DISC (GE) as in
    oracle.sim, B keeps its frame in USED with two dead pages."""
    t = _trace(2, 2, [("touch", [(0, 8, "W")]), ("discard", 0, 6, False)])
    o = replay_chunks(t, P, "eager")
    assert [ST_NAMES[x] for x in o.st] == ["GE", "G"]
    assert o.dead == [0, 0b0011]
    assert o.dump()["disc_order"] == [0] and o.dump()["used_order"] == [1]


# ------------------------------------------------------------------ reduction to oracle.sim
def _expand(tags, ppc):
    """Single-level content tags -> per-page tags of the same writes."""
    out = []
    for b, t in enumerate(tags):
        for p in range(ppc):
            q = b * ppc + p
            out.append(0 if t == 0 else ((t >> 32) << 32) | q)
    return out


def _aligned(t):
    """The same ops with every range widened (touch, prefetch, host_write) or narrowed
    (discard) to whole blocks: they cover the same blocks in oracle.sim's rules."""
    B = t.block_bytes
    tb = tg.TraceBuilder(B, t.arena_bytes, t.budget_bytes)
    out = lambda o, l: (o // B * B, (-(-(o + l) // B) - o // B) * B if l else 0)
    for (op, fl, off, ln, accs) in t.iter_ops():
        if op == tg.OP_TOUCH:
            tb.touch([(*out(a, l), k) for (a, l, k) in accs])
        elif op == tg.OP_PREFETCH:
            tb.prefetch(*out(off, ln), fl)
        elif op == tg.OP_DISCARD:
            lo, hi = -(-off // B), (off + ln) // B
            tb.discard(lo * B, max(0, hi - lo) * B, lazy_ok=bool(fl & tg.F_LAZY_OK))
        elif op == tg.OP_EVICT:
            tb.evict(ln)
        else:
            tb.host_write(*out(off, ln))
    return tb.build()


@settings(max_examples=120, deadline=None, suppress_health_check=[HealthCheck.too_slow])
@given(seed=hst.integers(0, 10**6), nblocks=hst.integers(1, 8), nframes=hst.integers(1, 4),
       ppc=hst.sampled_from([1, 2, 4]))
def test_reduces_to_single_level_without_partial_discards(seed, nblocks, nframes, ppc):
    """With every op chunk-granular, the page masks stay empty and the two-level model is
    oracle.sim: same states, queue orders and counters, and per-page contents = the
    chunk's writes."""
    raw = tg.gen_small(seed, nblocks=nblocks, nframes=nframes, n_ops=30)
    # one page per chunk is the single-level model whatever the ranges
    for t in ([_aligned(raw), raw] if ppc == 1 else [_aligned(raw)]):
        _same_as_single_level(t, ppc)


def _same_as_single_level(t, ppc):
    for mode in ("base", "eager", "lazy"):
        a = replay(t, mode).dump()
        b = replay_chunks(t, t.block_bytes // ppc, mode).dump()
        assert a["st"] == b["st"] and a["used_order"] == b["used_order"] and a["disc_order"] == b["disc_order"]
        assert a["stats"] == b["stats"]
        assert _expand(a["contents"], ppc) == b["contents"]
        assert not any(b["dead"])


# ------------------------------------------------------------------ page-level invariants
def _random_page_trace(seed, nchunks, nframes, n_ops=40):
    rng = np.random.default_rng(seed)
    npg = nchunks * PPC
    ops = []
    for _ in range(n_ops):
        r = rng.random()
        q = int(rng.integers(0, npg))
        n = int(rng.integers(1, min(6, npg - q) + 1))
        if r < 0.45:
            ops.append(("touch", [(q, n, "W" if rng.random() < 0.4 else "R")]))
        elif r < 0.7:
            ops.append(("discard", q, n, bool(rng.random() < 0.5)))
        elif r < 0.85:
            ops.append(("prefetch", q, n, tg.DST_GPU if rng.random() < 0.7 else tg.DST_HOST))
        else:
            ops.append(("evict", int(rng.integers(1, nframes + 1))))
    return _trace(nchunks, nframes, ops)


def _flat(t, mode):
    """Page-level semantic contract (§4.1): a write sets a page; a discard makes the
    fully covered pages don't-care until written again; a lazy one also until a prefetch
    precedes the write (A8, A17).  Sequence numbers follow the chunk model's sub-ops."""
    npg = t.nblocks * PPC
    val, dc, lazy = [0] * npg, [False] * npg, [False] * npg
    hist = [{0} for _ in range(npg)]
    seq = 0
    F = t.nframes
    for (op, fl, off, ln, accs) in t.iter_ops():
        if op == tg.OP_TOUCH:
            pages, wr = set(), set()
            for (a, l, k) in accs:
                r = range(a // P, (a + l - 1) // P + 1) if l else range(0)
                pages.update(r)
                if k & tg.ACC_WRITE:
                    wr.update(r)
            chunks = sorted({q // PPC for q in pages})
            for i in range(0, max(1, len(chunks)), F):
                seq += 1
                for c in chunks[i:i + F]:
                    for q in range(c * PPC, (c + 1) * PPC):
                        if q in wr:
                            v = (seq << 32) | q
                            hist[q].add(v)
                            if not lazy[q]:
                                val[q], dc[q] = v, False
        elif op == tg.OP_PREFETCH:
            pages = range(off // P, (off + ln - 1) // P + 1) if ln else range(0)
            nch = len({q // PPC for q in pages})
            seq += max(1, -(-nch // F)) if fl == tg.DST_GPU else 1
            for q in pages:
                lazy[q] = False
        elif op == tg.OP_DISCARD:
            seq += 1
            if mode == "base":
                continue
            for q in range(-(-off // P), (off + ln) // P):
                dc[q] = True
                if mode == "lazy" and (fl & tg.F_LAZY_OK):
                    lazy[q] = True
        else:
            seq += 1
    return val, dc, hist


@settings(max_examples=120, deadline=None, suppress_health_check=[HealthCheck.too_slow])
@given(seed=hst.integers(0, 10**6), nchunks=hst.integers(1, 6), nframes=hst.integers(1, 3))
def test_page_semantics_and_no_dead_transfers(seed, nchunks, nframes):
    """(iii)/(iv) per page; (ii) no D2H or H2D ever moves a dead page; conservation."""
    t = _random_page_trace(seed, nchunks, nframes)
    for mode in ("base", "eager", "lazy"):
        o = replay_chunks(t, P, mode, record=True)
        o.check_conservation()
        got = o.contents()
        val, dc, hist = _flat(t, mode)
        for q in range(len(got)):
            if not dc[q]:
                assert got[q] == val[q], (mode, q)
            else:
                assert got[q] in hist[q], (mode, q)
        if mode == "base":
            b = o.stats
            assert b["d2h_avoided_bytes"] == b["h2d_avoided_bytes"] == 0
