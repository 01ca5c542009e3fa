"""Pins of the CPU oracle against things other than itself (`-m "not gpu"`):
hand-enumerated scenarios (golden/scenarios.yaml), the C2 closed form, and the
textbook LRU / FIFO reductions (SURVEY.md §8(c) "What pins each part" 1-3)."""
from collections import OrderedDict, deque

import numpy as np
import pytest

import tracegen as tg
from oracle.sim import Oracle, replay, ST_NAMES, STAT_NAMES
import scenarios as scn

SCEN = scn.load()


@pytest.mark.parametrize("host_release", [True, False])
@pytest.mark.parametrize("name", sorted(SCEN))
def test_scenario(name, host_release):
    sc = SCEN[name]
    trace, mode = scn.build(sc)
    o = replay(trace, mode, host_release=host_release, overlap=sc.get("overlap", 0), reserve=sc.get("reserve", 0))
    o.check_conservation()
    d = o.dump()
    exp = sc["expect"]
    for k, v in exp["stats"].items():
        assert d["stats"][k] == v, (name, k, d["stats"][k], v)
    assert [ST_NAMES[s] for s in d["st"]] == exp["st"]
    if "used_order" in exp:
        assert d["used_order"] == exp["used_order"]
    if "disc_order" in exp:
        assert d["disc_order"] == exp["disc_order"]
    assert d["contents"] == scn.expected_contents(sc)


# --------------------------------------------------------------------- C2 closed form
@pytest.mark.parametrize("F,c,P", [(8, 2, 3), (16, 4, 4), (64, 8, 2), (4, 1, 5), (32, 16, 3), (6, 3, 2)])
@pytest.mark.parametrize("mode", ["base", "eager", "lazy"])
def test_c2_closed_form(F, c, P, mode):
    """SURVEY §8(c) item 2 (FIR-like stream, §7.2, Table 4):
    base: H2D = 2(P-1)F, D2H = (2P-1)F, ZF = 2F blocks; with discard: H2D = D2H = 0,
    ZF = 2PF; avoided = (4P-3)F blocks."""
    B = 4096
    t = tg.gen_c2(F, c, P, block_bytes=B)
    s = replay(t, mode).stats
    if mode == "base":
        assert (s["h2d_bytes"], s["d2h_bytes"], s["zf_bytes"]) == (2 * (P - 1) * F * B, (2 * P - 1) * F * B, 2 * F * B)
    else:
        assert (s["h2d_bytes"], s["d2h_bytes"], s["zf_bytes"]) == (0, 0, 2 * P * F * B)
        base = replay(t, "base").stats
        avoided = base["h2d_bytes"] + base["d2h_bytes"] - s["h2d_bytes"] - s["d2h_bytes"]
        assert avoided == (4 * P - 3) * F * B


def test_c2_fir_constant_savings():
    """Analogue of Table 4 (L397-403): under oversubscription every eviction writeback
    of a consumed window is redundant, and discard removes all of it.  Hand derivation
    (64-block buffer, 4-block chunks, P = 2 passes, budget F <= 32 blocks): base pass 1
    zero-fills 64 and writes back 64 - F; pass 2 migrates all 64 back and writes back
    64 -> avoided = (P*64 - F) + (P-1)*64 blocks; the discard run moves nothing."""
    B, P, total = 4096, 2, 64
    saved = []
    for F in (32, 16, 8):           # 200 %, 400 %, 800 % of the budget
        tb = tg.TraceBuilder(B, total * B, F * B)
        o, _ = tb.alloc("s", total * B)
        for j in range(P * (total // 4)):
            x = o + (j % (total // 4)) * 4 * B
            tb.prefetch(x, 4 * B, tg.DST_GPU)
            tb.touch([(x, 4 * B, tg.ACC_WRITE)])
            tb.discard(x, 4 * B, lazy_ok=True)
        t = tb.build()
        b, e = replay(t, "base").stats, replay(t, "eager").stats
        saved.append(b["h2d_bytes"] + b["d2h_bytes"] - e["h2d_bytes"] - e["d2h_bytes"])
        assert e["h2d_bytes"] == e["d2h_bytes"] == 0
    # every block's data is dead at discard time, so every base transfer is redundant;
    # D2H: all but the F resident blocks of the last pass are written back in every pass
    for F, s in zip((32, 16, 8), saved):
        assert s == ((P * total - F) + (P - 1) * total) * B


# --------------------------------------------------------------------- textbook reductions
def _lru_misses(seq, cap):
    c, misses, evict = OrderedDict(), 0, 0
    for x in seq:
        if x in c:
            c.move_to_end(x)
        else:
            misses += 1
            if len(c) == cap:
                c.popitem(last=False)
                evict += 1
            c[x] = 1
    return misses, evict, list(c)


def _fifo_misses(seq, cap):
    q, s, misses, evict = deque(), set(), 0, 0
    for x in seq:
        if x not in s:
            misses += 1
            if len(q) == cap:
                s.discard(q.popleft())
                evict += 1
            q.append(x)
            s.add(x)
    return misses, evict, list(q)


@pytest.mark.parametrize("seed", range(8))
@pytest.mark.parametrize("kind", ["prefetch", "touch"])
def test_textbook_cache(seed, kind):
    """Discard-free single-block ops: prefetch-only = LRU cache (prefetch moves a page to
    the MRU side, L217); touch-only = FIFO cache (recency is set only at fault time, A1)."""
    rng = np.random.default_rng(seed)
    nb, F, B = 12, int(rng.integers(1, 6)), 4096
    seq = [int(x) for x in rng.integers(0, nb, size=300)]
    tb = tg.TraceBuilder(B, nb * B, F * B)
    for x in seq:
        if kind == "prefetch":
            tb.prefetch(x * B, B, tg.DST_GPU)
        else:
            tb.touch([(x * B, B, tg.ACC_READ)])
    o = replay(tb.build(), "base")
    misses, evict, order = (_lru_misses if kind == "prefetch" else _fifo_misses)(seq, F)
    s = o.stats
    assert (s["h2d_bytes"] + s["zf_bytes"]) // B == misses
    assert s["d2h_bytes"] // B == evict == s["evictions"]
    assert o.dump()["used_order"] == order


def test_invalid_range_rejected_without_effect():
    o = Oracle(4096, 4 * 4096, 2 * 4096)
    with pytest.raises(ValueError):
        o.prefetch(3 * 4096, 2 * 4096, 0)
    with pytest.raises(ValueError):
        o.touch([(0, 4096, 1), (4 * 4096, 1, 1)])
    assert o.clock == 0 and all(v == 0 for v in o.stats.values())


def test_subop_split_ascending():
    """A3: an op with more distinct blocks than frames is split into ascending sub-ops
    of <= nframes blocks, each with its own seq; blocks of the current sub-op are never
    victims.  1 frame, touch 3 blocks W: each block is zero-filled, then evicted by the
    next sub-op; the last stays resident."""
    B = 4096
    tb = tg.TraceBuilder(B, 3 * B, 1 * B)
    tb.touch([(0, 3 * B, tg.ACC_WRITE)])
    o = replay(tb.build(), "eager")
    d = o.dump()
    assert d["stats"]["subops"] == 3 and d["stats"]["ops"] == 1
    assert [ST_NAMES[s] for s in d["st"]] == ["H", "H", "G"]
    assert d["contents"] == [(1 << 32) | 0, (2 << 32) | 1, (3 << 32) | 2]
    assert d["stats"]["d2h_bytes"] == 2 * B and d["stats"]["zf_bytes"] == 3 * B


def test_stat_names_match_abi_order():
    """um_stats field order in include/um.h (the ABI the CUDA side implements)."""
    import re, os
    h = open(os.path.join(os.path.dirname(__file__), "..", "include", "um.h")).read()
    body = re.search(r"typedef struct\s*\{([^}]*)\}\s*um_stats;", h).group(1)
    names = re.findall(r"\b([a-z0-9_]+)\s*[,;]", body.replace("int64_t", ""))
    assert tuple(n for n in names if not n.startswith("pad")) == STAT_NAMES


@pytest.mark.parametrize("nb,p", [(8, 0.0), (8, 0.5), (16, 1.0), (10, 0.3)])
@pytest.mark.parametrize("pressure", [False, True])
@pytest.mark.parametrize("mode", ["eager", "lazy"])
def test_c4_closed_form(nb, p, pressure, mode):
    """C4 by hand.  nb resident written blocks are discarded, then
    k = round(p*nb) are re-touched (prefetch + write).
    No pressure: the pages are still resident -> k remaps (UvmDiscard re-maps, §5.7
    L229) or k revalidations (UvmDiscardLazy's prefetch sets the dirty bits, L190); no
    transfer, no extra zeroing.
    Pressure (a filler of nb blocks prefetched in between, budget = nb): all nb discarded
    pages are reclaimed first (discarded FIFO, L221) with no write-back (d2h_avoided =
    nb); the re-touch zero-fills k blocks instead of migrating them (h2d_avoided = k,
    L200) and evicts the k LRU filler blocks, which are valid and written back (A10)."""
    B = 4096
    t = tg.gen_c4(nb * B, p, block_bytes=B, pressure=pressure)
    k = int(round(p * nb))
    s = replay(t, mode).stats
    if not pressure:
        assert s["zf_bytes"] == nb * B and s["h2d_bytes"] == s["d2h_bytes"] == 0
        assert (s["remaps"], s["revalidations"]) == ((k, 0) if mode == "eager" else (0, k))
        assert s["unmaps"] == (nb if mode == "eager" else 0)
    else:
        assert s["zf_bytes"] == (2 * nb + k) * B
        assert s["d2h_avoided_bytes"] == nb * B and s["h2d_avoided_bytes"] == k * B
        assert s["d2h_bytes"] == k * B and s["h2d_bytes"] == 0
        assert s["remaps"] == s["revalidations"] == 0
        assert s["unmaps"] == nb          # eager: at discard; lazy: at reclaim (§5.6)
        assert s["evictions"] == nb + k


def test_sparse_trace_shape():
    """gen_sparse must produce what the fault-list path needs (sorted, disjoint batches
    of more than kIvInline = 24 records whose merged runs average <= 3 blocks), or the
    GPU test of that path would silently exercise the interval form instead."""
    t = tg.gen_sparse(0)
    B = t.block_bytes
    seen = 0
    for (op, _fl, _off, _ln, accs) in t.iter_ops():
        if op != tg.OP_TOUCH:
            continue
        lo = [a // B for (a, _l, _k) in accs]
        assert lo == sorted(set(lo)) and len(lo) > 24
        runs = 1 + sum(1 for x, y in zip(lo, lo[1:]) if y != x + 1)
        assert len(lo) <= 3 * runs
        seen += 1
    assert seen >= 5


@pytest.mark.parametrize("mode", ["base", "eager", "lazy"])
def test_free_releases_without_transfers(mode):
    """R9 (um_free): after the hash join frees its intermediates and outputs they are U
    (contents zero); the frames they held are reused with no write-back, so freeing
    never adds a transfer; conservation holds throughout."""
    B = 64 << 10
    kw = dict(block_bytes=B, budget_bytes=(36 << 20) // B * B, table_bytes=8 << 20)
    a = replay(tg.gen_hashjoin(**kw), mode)
    t = tg.gen_hashjoin(free_at_end=True, **kw)
    b = replay(t, mode)
    b.check_conservation()
    for name, (off, ln) in t.buffers.items():
        blocks = range(off // B, (off + ln) // B)
        if name in ("R", "S"):
            assert all(ST_NAMES[b.st[x]] != "U" for x in blocks)
        else:
            assert all(ST_NAMES[b.st[x]] == "U" and b.content(x) == 0 for x in blocks)
    # the freed blocks' frames serve the final read of the tables: no more write-backs
    # than the same run without the free and one more read
    assert b.stats["d2h_bytes"] == a.stats["d2h_bytes"] and b.stats["evictions"] == a.stats["evictions"]


def test_slice_ops_drops_private_meta():
    """A sub-trace must not inherit a consumer's cache of its parent's op list."""
    t = tg.gen_c1(0)
    t.meta["_calls_eager"] = ["stale"]
    s = t.slice_ops(0, 10)
    assert "_calls_eager" not in s.meta and len(s) == 10 and s.meta["seed"] == 0


# --------------------------------------------------------------------- state microbench closed form
@pytest.mark.parametrize("nb,nf,n,seed", [(4096, 2730, 2048, 0), (4096, 2200, 2048, 1), (60000, 40000, 30000, 2)])
def test_state_micro_closed_form(nb, nf, n, seed):
    """The state microbench's sequence (tracegen.gen_state_micro: touch of n random blocks,
    discard [0, n), touch of n other random blocks) derived by hand from §8(c)'s sub-op
    algorithm with set arithmetic: the first touch zero-fills all n (free frames suffice);
    the discard unmaps the G blocks inside [0, n) into DISC in ascending order (§5.1);
    the second touch revives the discarded blocks it covers (§5.7), hits the other
    resident ones, zero-fills the rest, and reclaims k = need - free victims: the head of
    DISC without a transfer, then (if DISC runs out) the LRU end of USED -- the first
    touch's blocks outside [0, n), ascending -- written back (§5.5)."""
    B = 4096
    t = tg.gen_state_micro(seed, block_bytes=B, arena_bytes=nb * B, budget_bytes=nf * B, n=n)
    b0 = set((t.acc["off"][:n] // B).tolist())
    b1 = set((t.acc["off"][n:] // B).tolist())
    ge = sorted(b for b in b0 if b < n)
    need = len(b1 - b0)
    free = nf - n
    k = max(0, need - free)
    cand = [b for b in ge if b not in b1]      # DISC head first, skipping the pinned sub-op
    ucand = sorted(b0 - set(ge) - b1)          # then USED: (ukey = 1, block) ascending
    vd = cand[:k]
    vu = ucand[:k - len(vd)]
    assert len(vd) + len(vu) == k
    o = replay(t, "eager")
    s = o.stats
    assert s["zf_bytes"] == (n + need) * B
    assert s["unmaps"] == len(ge)
    assert s["remaps"] == len(b1 & set(ge))
    assert s["hits"] == len(b1 & (b0 - set(ge)))
    assert s["faults"] == n + need + len(b1 & set(ge))
    assert s["evictions"] == k
    assert s["d2h_avoided_bytes"] == len(vd) * B and s["d2h_bytes"] == len(vu) * B and s["h2d_bytes"] == 0
    st = o.st
    assert all(st[v] == 2 for v in vd) and all(st[v] == 1 for v in vu)        # HD, H
    assert sorted(b for b in range(nb) if st[b] == 4) == sorted(set(cand) - set(vd))   # GE left
    assert list(o.disc) == [b for b in cand if b not in set(vd)]
