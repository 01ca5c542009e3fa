"""Brute force and invariants for the oracle.

`LinkedModel` below is a SECOND, independently written formulation of the same paper
model: explicit doubly-linked page queues (§5.5) with head/tail pointers, state
names as strings, and per-op transition tables.  It shares nothing with oracle/sim.py
except the trace it reads.  Exhaustive enumeration over tiny configurations and random
traces must give identical states, queue orders, counters and contents.
"""
import itertools

import numpy as np
import pytest
from hypothesis import given, settings, strategies as hst, HealthCheck

import tracegen as tg
from oracle.sim import G, Oracle, apply_op, replay, ST_NAMES


class _Node:
    __slots__ = ("blk", "prev", "next")

    def __init__(self, blk):
        self.blk, self.prev, self.next = blk, None, None


class _DList:
    def __init__(self):
        self.head = self.tail = None
        self.where = {}

    def push_tail(self, blk):
        n = _Node(blk)
        n.prev = self.tail
        if self.tail:
            self.tail.next = n
        else:
            self.head = n
        self.tail = n
        self.where[blk] = n

    def remove(self, blk):
        n = self.where.pop(blk)
        if n.prev:
            n.prev.next = n.next
        else:
            self.head = n.next
        if n.next:
            n.next.prev = n.prev
        else:
            self.tail = n.prev

    def __iter__(self):
        n = self.head
        while n:
            yield n.blk
            n = n.next

    def __contains__(self, blk):
        return blk in self.where


class LinkedModel:
    """Independent re-statement of the transition table."""

    def __init__(self, B, nblocks, nframes, mode, host_release=True, overlap=0):
        self.B, self.n, self.F, self.mode, self.rel = B, nblocks, nframes, mode, host_release
        # R7 window: block lists of the previous GPU sub-ops, newest first
        self.W, self.recent = overlap, []
        self.state = ["U"] * nblocks
        self.gpu = [0] * nblocks
        self.host = [0] * nblocks
        self.used, self.disc = _DList(), _DList()
        self.nfree = nframes
        self.t = 0
        self.c = {k: 0 for k in ("h2d_bytes", "d2h_bytes", "zf_bytes", "h2d_avoided_bytes",
                                 "d2h_avoided_bytes", "faults", "hits", "remaps", "unmaps",
                                 "revalidations", "refreshes", "evictions", "ops", "subops")}

    def tick(self):
        self.t += 1
        self.c["subops"] += 1
        return self.t

    def evict_one(self, exclude):
        for q in (self.disc, self.used):
            for blk in q:
                if blk not in exclude:
                    return blk
        return None

    def reclaim(self, v):
        s = self.state[v]
        if s == "G":
            self.host[v] = self.gpu[v]
            self.c["d2h_bytes"] += self.B
            self.used.remove(v)
            self.state[v] = "H"
        else:
            self.c["d2h_avoided_bytes"] += self.B
            self.c["unmaps"] += 1 if s == "GL" else 0
            self.disc.remove(v)
            self.state[v] = "HD"
        self.c["evictions"] += 1
        self.nfree += 1

    def gpu_sub(self, blocks, touch, writes):
        t = self.tick()
        excl = set(blocks)
        if self.W:
            # protect previous sub-ops newest first while the frames they could hold,
            # plus this sub-op's, fit in the budget (R7)
            room = self.F - len(blocks)
            for prev in self.recent[:self.W]:
                room -= len(prev)
                if room < 0:
                    break
                excl.update(prev)
            self.recent.insert(0, list(blocks))
        while sum(1 for b in blocks if self.state[b] in ("U", "H", "HD")) > self.nfree:
            # one victim at a time, each time re-scanning from the queue heads
            self.reclaim(self.evict_one(excl))
        for b in blocks:
            s = self.state[b]
            if s in ("U", "H", "HD"):
                self.nfree -= 1
                if s == "H":
                    self.gpu[b] = self.host[b]
                    self.c["h2d_bytes"] += self.B
                    if self.rel:
                        self.host[b] = 0
                else:
                    self.gpu[b] = 0
                    self.c["zf_bytes"] += self.B
                    if s == "HD":
                        self.c["h2d_avoided_bytes"] += self.B
                self.c["faults"] += touch
                self.state[b] = "G"
                self.used.push_tail(b)
            elif s == "G":
                if touch:
                    self.c["hits"] += 1
                else:
                    self.c["refreshes"] += 1
                    self.used.remove(b)
                    self.used.push_tail(b)
            elif s == "GE":
                self.c["remaps"] += 1
                self.c["faults"] += touch
                self.disc.remove(b)
                self.state[b] = "G"
                self.used.push_tail(b)
            elif s == "GL":
                if touch:
                    self.c["hits"] += 1
                else:
                    self.c["revalidations"] += 1
                    self.disc.remove(b)
                    self.state[b] = "G"
                    self.used.push_tail(b)
        for b in blocks:
            if b in writes:
                self.gpu[b] = (t << 32) | b

    def run(self, trace):
        B = self.B
        for (op, fl, off, ln, accs) in trace.iter_ops():
            self.c["ops"] += 1
            if op == tg.OP_TOUCH:
                blk, wr = set(), set()
                for (a, l, k) in accs:
                    if l:
                        r = range(a // B, (a + l - 1) // B + 1)
                        blk.update(r)
                        if k & tg.ACC_WRITE:
                            wr.update(r)
                s = sorted(blk)
                parts = [s[i:i + self.F] for i in range(0, len(s), self.F)] or [[]]
                for p in parts:
                    self.gpu_sub(p, 1, wr)
            elif op == tg.OP_PREFETCH and fl == tg.DST_GPU:
                s = list(range(off // B, (off + ln - 1) // B + 1)) if ln else []
                parts = [s[i:i + self.F] for i in range(0, len(s), self.F)] or [[]]
                for p in parts:
                    self.gpu_sub(p, 0, set())
            elif op == tg.OP_PREFETCH:
                self.tick()
                for b in (range(off // B, (off + ln - 1) // B + 1) if ln else []):
                    s = self.state[b]
                    if s == "G":
                        self.host[b] = self.gpu[b]
                        self.c["d2h_bytes"] += B
                        self.used.remove(b)
                        self.nfree += 1
                    elif s in ("GE", "GL"):
                        self.c["d2h_avoided_bytes"] += B
                        self.c["unmaps"] += s == "GL"
                        self.disc.remove(b)
                        self.nfree += 1
                    self.state[b] = "H"
            elif op == tg.OP_DISCARD:
                t = self.tick()
                if self.mode == "base":
                    continue
                lazy = self.mode == "lazy" and (fl & tg.F_LAZY_OK)
                lo, hi = -(-off // B), (off + ln) // B
                table = ({"G": "GL", "H": "HD"} if lazy else {"G": "GE", "GL": "GE", "H": "HD"})
                for b in range(lo, hi):
                    s = self.state[b]
                    if s not in table:
                        continue
                    if s == "G":
                        self.used.remove(b)
                        self.disc.push_tail(b)
                    if s in ("G", "GL") and not lazy:
                        self.c["unmaps"] += 1
                    if s == "H" and self.rel:
                        self.host[b] = 0
                    self.state[b] = table[s]
            elif op == tg.OP_EVICT:
                self.tick()
                k = -(-ln // B) - self.nfree
                while k > 0:
                    v = self.evict_one(())
                    if v is None:
                        break
                    self.reclaim(v)
                    k -= 1
            elif op == tg.OP_HOST_WRITE:
                t = self.tick()
                for b in (range(off // B, (off + ln - 1) // B + 1) if ln else []):
                    assert self.state[b] == "H"
                    self.host[b] = (t << 32) | b
        return self

    def result(self):
        content = [self.gpu[b] if s in ("G", "GE", "GL") else (self.host[b] if s in ("H", "HD") else 0)
                   for b, s in enumerate(self.state)]
        return {"st": list(self.state), "used_order": list(self.used), "disc_order": list(self.disc),
                "stats": dict(self.c), "contents": content}


def _compare(trace, mode, host_release=True, overlap=0):
    o = replay(trace, mode, host_release=host_release, overlap=overlap)
    o.check_conservation()
    d = o.dump()
    m = LinkedModel(trace.block_bytes, trace.nblocks, trace.nframes, mode, host_release,
                    overlap).run(trace).result()
    assert [ST_NAMES[s] for s in d["st"]] == m["st"]
    assert d["used_order"] == m["used_order"]
    assert d["disc_order"] == m["disc_order"]
    assert d["stats"] == m["stats"]
    assert d["contents"] == m["contents"]
    return d


# ------------------------------------------------------------------ exhaustive enumeration
B0 = 4096
_ALPHA = (
    [("touch", b, k) for b in range(3) for k in (tg.ACC_READ, tg.ACC_WRITE)]
    + [("touch2", 0, tg.ACC_WRITE), ("touch3", 0, tg.ACC_WRITE)]
    + [("pf", b, d) for b in range(3) for d in (tg.DST_GPU, tg.DST_HOST)]
    + [("disc", b, lz) for b in range(3) for lz in (0, 1)]
    + [("evict", 1, 0)]
)


def _mk(seq, nframes):
    tb = tg.TraceBuilder(B0, 3 * B0, nframes * B0)
    for (op, b, x) in seq:
        if op == "touch":
            tb.touch([(b * B0, B0, x)])
        elif op == "touch2":
            tb.touch([(0, B0, x), (B0 + 100, B0, tg.ACC_READ)])     # blocks 0-2, overlapping ranges
        elif op == "touch3":
            tb.touch([(0, 3 * B0, x)])
        elif op == "pf":
            tb.prefetch(b * B0, B0, x)
        elif op == "disc":
            tb.discard(b * B0, B0, lazy_ok=bool(x))
        elif op == "evict":
            tb.evict(B0)
    return tb.build()


@pytest.mark.parametrize("overlap", [0, 2])
@pytest.mark.parametrize("nframes", [1, 2])
@pytest.mark.parametrize("length", [1, 2, 3])
def test_exhaustive_vs_linked_model(nframes, length, overlap):
    n = 0
    for seq in itertools.product(_ALPHA, repeat=length):
        t = _mk(seq, nframes)
        for mode in ("base", "eager", "lazy"):
            _compare(t, mode, overlap=overlap)
        n += 1
    assert n == len(_ALPHA) ** length


@pytest.mark.slow
@pytest.mark.parametrize("nframes", [1, 2])
def test_exhaustive_len4_sampled(nframes):
    rng = np.random.default_rng(nframes)
    for _ in range(3000):
        seq = [_ALPHA[i] for i in rng.integers(0, len(_ALPHA), size=4)]
        t = _mk(seq, nframes)
        for mode in ("base", "eager", "lazy"):
            _compare(t, mode)


# ------------------------------------------------------------------ random traces
@settings(max_examples=150, deadline=None, suppress_health_check=[HealthCheck.too_slow])
@given(seed=hst.integers(0, 10**6), nblocks=hst.integers(1, 8), nframes=hst.integers(1, 4),
       host_release=hst.booleans())
def test_random_vs_linked_model(seed, nblocks, nframes, host_release):
    t = tg.gen_small(seed, nblocks=nblocks, nframes=nframes, n_ops=30)
    for mode in ("base", "eager", "lazy"):
        _compare(t, mode, host_release)


@pytest.mark.parametrize("seed", range(3))
def test_c1_vs_linked_model(seed):
    t = tg.gen_c1(seed).slice_ops(0, 3000)
    for mode in ("base", "eager", "lazy"):
        _compare(t, mode)


# ------------------------------------------------------------------ invariants (i)-(vii)
def _strip_discards(trace):
    keep = trace.ops["op"] != tg.OP_DISCARD
    idx = np.nonzero(keep)[0]
    parts = [trace.slice_ops(int(i), int(i) + 1) for i in idx]
    tb = tg.TraceBuilder(trace.block_bytes, trace.arena_bytes, trace.budget_bytes)
    for p in parts:
        for (o, fl, off, ln, accs) in p.iter_ops():
            if o == tg.OP_TOUCH:
                tb.touch(accs)
            elif o == tg.OP_PREFETCH:
                tb.prefetch(off, ln, fl)
            elif o == tg.OP_EVICT:
                tb.evict(ln)
            elif o == tg.OP_HOST_WRITE:
                tb.host_write(off, ln)
    return tb.build()


@settings(max_examples=60, deadline=None)
@given(seed=hst.integers(0, 10**6), nblocks=hst.integers(2, 10), nframes=hst.integers(1, 4))
def test_inv_i_base_equals_no_discard(seed, nblocks, nframes):
    """(i) Base mode == the same trace with its discard ops removed (state, order,
    transfer counters; seqs differ so contents are not compared)."""
    t = tg.gen_small(seed, nblocks=nblocks, nframes=nframes, n_ops=40)
    a, b = replay(t, "base").dump(), replay(_strip_discards(t), "base").dump()
    assert a["st"] == b["st"] and a["used_order"] == b["used_order"] and a["disc_order"] == b["disc_order"]
    for k in a["stats"]:
        if k not in ("ops", "subops"):
            assert a["stats"][k] == b["stats"][k], k


@settings(max_examples=60, deadline=None)
@given(seed=hst.integers(0, 10**6), nblocks=hst.integers(2, 10), nframes=hst.integers(1, 4))
def test_inv_ii_no_writeback_of_discarded(seed, nblocks, nframes):
    """(ii) No D2H ever moves a block in GE/GL/HD; no H2D ever moves one in HD (the two
    RMT directions of Fig. 2 (6)(7), L131)."""
    t = tg.gen_small(seed, nblocks=nblocks, nframes=nframes, n_ops=40)
    for mode in ("eager", "lazy"):
        o = replay(t, mode, record=True)
        for (seq, kind, b, prev) in o.log:
            if kind == "D2H":
                assert ST_NAMES[prev] == "G"
            if kind == "H2D":
                assert ST_NAMES[prev] == "H"


class FlatMemory:
    """(iii)/(iv) The semantic contract of §4.1 (L160) on a flat array: writes set a
    block's value; an eager discard makes it don't-care until the next write; a lazy
    discard stays don't-care until a prefetch (either destination, A17) precedes the
    next write (A8)."""

    def __init__(self, trace, mode):
        self.t, self.mode = trace, mode

    def run(self):
        t, B, F = self.t, self.t.block_bytes, self.t.nframes
        val = [0] * t.nblocks
        dc = [False] * t.nblocks           # don't-care
        lazy_pending = [False] * t.nblocks  # lazily discarded, no prefetch since
        history = [{0} for _ in range(t.nblocks)]
        seq = 0
        for (op, fl, off, ln, accs) in t.iter_ops():
            if op == tg.OP_TOUCH:
                blk, wr = set(), set()
                for (a, l, k) in accs:
                    if l:
                        r = range(a // B, (a + l - 1) // B + 1)
                        blk.update(r)
                        if k & tg.ACC_WRITE:
                            wr.update(r)
                s = sorted(blk)
                for i in range(0, max(1, len(s)), F):
                    seq += 1
                    for b in s[i:i + F]:
                        if b in wr:
                            v = (seq << 32) | b
                            history[b].add(v)
                            if lazy_pending[b]:
                                continue            # write may be lost (A8)
                            val[b], dc[b] = v, False
            elif op == tg.OP_PREFETCH:
                n = -(-len(range(off // B, (off + ln - 1) // B + 1)) // F) if (fl == tg.DST_GPU and ln) else 1
                seq += n
                for b in (range(off // B, (off + ln - 1) // B + 1) if ln else []):
                    lazy_pending[b] = False
            elif op == tg.OP_DISCARD:
                seq += 1
                if self.mode == "base":
                    continue
                for b in range(-(-off // B), (off + ln) // B):
                    dc[b] = True
                    if self.mode == "lazy" and (fl & tg.F_LAZY_OK):
                        lazy_pending[b] = True
            elif op == tg.OP_EVICT:
                seq += 1
            elif op == tg.OP_FREE:
                # R9: fully covered blocks are released and read as never populated (zeros)
                seq += 1
                for b in range(-(-off // B), (off + ln) // B):
                    val[b], dc[b], lazy_pending[b] = 0, False, False
                    history[b].add(0)
            elif op == tg.OP_HOST_WRITE:
                seq += 1
                for b in (range(off // B, (off + ln - 1) // B + 1) if ln else []):
                    v = (seq << 32) | b
                    history[b].add(v)
                    val[b], dc[b], lazy_pending[b] = v, False, False
        return val, dc, history


@settings(max_examples=80, deadline=None)
@given(seed=hst.integers(0, 10**6), nblocks=hst.integers(2, 10), nframes=hst.integers(1, 4),
       host_release=hst.booleans())
def test_inv_iii_iv_flat_memory(seed, nblocks, nframes, host_release):
    t = tg.gen_small(seed, nblocks=nblocks, nframes=nframes, n_ops=40)
    for mode in ("base", "eager", "lazy"):
        got = replay(t, mode, host_release=host_release).contents()
        val, dc, hist = FlatMemory(t, mode).run()
        for b in range(t.nblocks):
            if not dc[b]:
                assert got[b] == val[b], (mode, b)          # (iii)
            else:
                assert got[b] in hist[b], (mode, b)         # (iv): 0 or an earlier stamp


@pytest.mark.parametrize("seed", range(4))
def test_inv_iii_c1(seed):
    t = tg.gen_c1(seed).slice_ops(0, 4000)
    for mode in ("base", "eager", "lazy"):
        got = replay(t, mode).contents()
        val, dc, hist = FlatMemory(t, mode).run()
        assert all(got[b] == val[b] for b in range(t.nblocks) if not dc[b])
        assert all(got[b] in hist[b] for b in range(t.nblocks) if dc[b])


@settings(max_examples=60, deadline=None)
@given(seed=hst.integers(0, 10**6), nblocks=hst.integers(1, 6))
def test_inv_v_no_pressure(seed, nblocks):
    """(v) arena <= budget: base and discard modes move the same H2D/D2H bytes (the equal
    <100 % columns of Tables 4/6/8, L397-463), for traces without evict, without
    prefetch(HOST) of discarded blocks and without discards of host-resident blocks."""
    t = tg.gen_small(seed, nblocks=nblocks, nframes=nblocks, n_ops=40, mix=[55, 25, 0, 10, 10, 0, 0])
    s = {m: replay(t, m).stats for m in ("base", "eager", "lazy")}
    for m in ("eager", "lazy"):
        assert s[m]["h2d_bytes"] == s["base"]["h2d_bytes"]
        assert s[m]["d2h_bytes"] == s["base"]["d2h_bytes"]
        assert s[m]["evictions"] == 0


@pytest.mark.parametrize("which", ["c2", "c3small", "c4"])
def test_inv_vi_eager_equals_lazy(which):
    """(vi) With every discard lazy_ok (each reuse preceded by a prefetch), eager and lazy
    give identical H2D/D2H/ZF bytes (Tables 4/6/8: within 0.4 %, L397-463)."""
    if which == "c2":
        t = tg.gen_c2(16, 4, 3, block_bytes=4096)
    elif which == "c3small":
        t = tg.gen_c3(block_bytes=64 * 1024, budget_bytes=96 * 1024 * 1024, iterations=2,
                      workspace_bytes=1 << 20, layers=tg.scale_layers(tg.VGG16, 1.0 / 4096, 1.0 / 64), batch=32)
    else:
        t = tg.gen_c4(4 << 20, 0.5, block_bytes=64 * 1024, pressure=True)
    assert tg.check_lazy_ok(t) == []
    e, l = replay(t, "eager").stats, replay(t, "lazy").stats
    for k in ("h2d_bytes", "d2h_bytes", "zf_bytes", "h2d_avoided_bytes", "d2h_avoided_bytes", "evictions"):
        assert e[k] == l[k], k


@pytest.mark.parametrize("seed", range(3))
def test_inv_vii_conservation_every_op(seed):
    from oracle.sim import Oracle, apply_op
    t = tg.gen_small(seed, nblocks=8, nframes=3, n_ops=200)
    for mode in ("base", "eager", "lazy"):
        o = Oracle(t.block_bytes, t.arena_bytes, t.budget_bytes, discard_off=(mode == "base"))
        for op in t.iter_ops():
            apply_op(o, op, mode)
            o.check_conservation()


def test_host_release_changes_only_discarded_contents():
    """Reading R1 (host copy released when a block leaves H) changes no counter, state
    or queue, and only contents of blocks whose value §4.1 leaves open."""
    for seed in range(20):
        t = tg.gen_small(seed, nblocks=8, nframes=3, n_ops=60)
        for mode in ("base", "eager", "lazy"):
            a, b = replay(t, mode, host_release=True).dump(), replay(t, mode, host_release=False).dump()
            assert a["stats"] == b["stats"] and a["st"] == b["st"]
            assert a["used_order"] == b["used_order"] and a["disc_order"] == b["disc_order"]
            val, dc, _ = FlatMemory(t, mode).run()
            for x in range(t.nblocks):
                if not dc[x]:
                    assert a["contents"][x] == b["contents"][x]


@pytest.mark.parametrize("ov", [0.8, 2, 3, 4])
def test_next3_radix_hashjoin_invariants(ov):
    """NEXT-3 workloads (radix sort §7.3, hash join §7.4): lazy_ok discards are valid;
    eager and lazy move identical bytes (vi); without pressure discard changes no
    transfer (v; the equal <100 % columns of Tables 6 and 8); under pressure discard
    never increases H2D+D2H."""
    MiB = 1 << 20
    B = 64 * 1024
    traces = [tg.gen_radix(block_bytes=B, budget_bytes=int(64 * MiB / ov) // B * B, data_bytes=32 * MiB),
              tg.gen_hashjoin(block_bytes=B, budget_bytes=int(72 * MiB / ov) // B * B, table_bytes=8 * MiB)]
    for t in traces:
        assert tg.check_lazy_ok(t) == []
        s = {m: replay(t, m).stats for m in ("base", "eager", "lazy")}
        for k in ("h2d_bytes", "d2h_bytes", "zf_bytes"):
            assert s["eager"][k] == s["lazy"][k]
        mv = {m: s[m]["h2d_bytes"] + s[m]["d2h_bytes"] for m in s}
        if ov < 1:
            assert mv["eager"] == mv["base"]
        else:
            assert mv["eager"] <= mv["base"]


# ------------------------------------------------------------------ R7 (UM_F_OVERLAP)
@settings(max_examples=150, deadline=None, suppress_health_check=[HealthCheck.too_slow])
@given(seed=hst.integers(0, 10**6), nblocks=hst.integers(1, 10), nframes=hst.integers(1, 5),
       overlap=hst.integers(1, 3))
def test_overlap_vs_linked_model(seed, nblocks, nframes, overlap):
    """The window rule (reading R7) restated independently in the linked-list model; its
    victim loop fails if the window ever leaves fewer candidates than k."""
    t = tg.gen_small(seed, nblocks=nblocks, nframes=nframes, n_ops=40)
    for mode in ("base", "eager", "lazy"):
        _compare(t, mode, overlap=overlap)


@settings(max_examples=60, deadline=None)
@given(seed=hst.integers(0, 10**6), nblocks=hst.integers(2, 10), nframes=hst.integers(1, 4))
def test_overlap_keeps_semantics(seed, nblocks, nframes):
    """R7 changes which block is evicted, never what a program reads: the flat-memory
    check (iii)/(iv) and the no-writeback-of-discarded invariant (ii) hold with the
    window, and without memory pressure the window changes nothing at all."""
    t = tg.gen_small(seed, nblocks=nblocks, nframes=nframes, n_ops=40)
    for mode in ("base", "eager", "lazy"):
        o = replay(t, mode, overlap=2, record=True)
        o.check_conservation()
        got = o.contents()
        val, dc, hist = FlatMemory(t, mode).run()
        for b in range(t.nblocks):
            assert got[b] == val[b] if not dc[b] else got[b] in hist[b], (mode, b)
        for (_s, kind, _b, prev) in o.log:
            if kind == "D2H":
                assert ST_NAMES[prev] == "G"
    roomy = tg.gen_small(seed, nblocks=nblocks, nframes=nblocks, n_ops=40)   # arena <= budget
    for mode in ("base", "eager", "lazy"):
        assert replay(roomy, mode, overlap=2).dump() == replay(roomy, mode).dump()


@settings(max_examples=80, deadline=None)
@given(seed=hst.integers(0, 10**6), nblocks=hst.integers(2, 10), nframes=hst.integers(1, 4),
       host_release=hst.booleans())
def test_free_flat_memory_and_conservation(seed, nblocks, nframes, host_release):
    """R9 (um_free) inside random traces: conservation after every op, the flat-memory
    contract with a free reading back as zeros, and no discarded block written back."""
    t = tg.gen_small(seed, nblocks=nblocks, nframes=nframes, n_ops=50, mix=[45, 12, 5, 10, 10, 3, 2, 13])
    for mode in ("base", "eager", "lazy"):
        o = Oracle(t.block_bytes, t.arena_bytes, t.budget_bytes, discard_off=(mode == "base"),
                   host_release=host_release, record=True)
        for op in t.iter_ops():
            apply_op(o, op, mode)
            o.check_conservation()
        assert all(k != "D2H" or p == G for (_s, k, _b, p) in o.log)
        val, dc, hist = FlatMemory(t, mode).run()
        got = o.contents()
        for b in range(t.nblocks):
            if not dc[b]:
                assert got[b] == val[b], (mode, b)
            else:
                assert got[b] in hist[b], (mode, b)


# ------------------------------------------------------------------ R12 (proactive eviction)
@settings(max_examples=80, deadline=None)
@given(seed=hst.integers(0, 10**6), nblocks=hst.integers(2, 10), nframes=hst.integers(1, 5),
       reserve=hst.integers(1, 4), overlap=hst.sampled_from([0, 2]))
def test_reserve_keeps_semantics(seed, nblocks, nframes, reserve, overlap):
    """R12 changes when a block is evicted, never what a program reads: the flat-memory
    check (iii)/(iv), conservation after every op and the no-writeback-of-discarded
    invariant (ii) hold; after a GPU op of at most nframes blocks without the window,
    either `reserve` frames are free or every queued block belongs to that op (only the
    op's own blocks are kept from early reclaim); with room to spare it changes nothing."""
    t = tg.gen_small(seed, nblocks=nblocks, nframes=nframes, n_ops=40)
    for mode in ("base", "eager", "lazy"):
        o = Oracle(t.block_bytes, t.arena_bytes, t.budget_bytes, discard_off=(mode == "base"),
                   record=True, overlap=overlap, reserve=reserve)
        for op in t.iter_ops():
            apply_op(o, op, mode)
            o.check_conservation()
            kind, flags, off, ln, accs = op
            gpu = kind == 0 or (kind == 1 and flags == 0)
            if gpu and not overlap:
                cover = set()
                for (a, n, _k) in (accs if kind == 0 else [(off, ln, 0)]):
                    cover.update(o._cover(a, n))
                if 0 < len(cover) <= nframes:
                    others = [b for b in list(o.used) + list(o.disc) if b not in cover]
                    assert o.free >= reserve or not others, (mode, o.free, others)
        assert all(k != "D2H" or p == G for (_s, k, _b, p) in o.log)
        val, dc, hist = FlatMemory(t, mode).run()
        got = o.contents()
        for b in range(t.nblocks):
            assert got[b] == val[b] if not dc[b] else got[b] in hist[b], (mode, b)
    roomy = tg.gen_small(seed, nblocks=nblocks, nframes=nblocks + reserve, n_ops=40)
    for mode in ("base", "eager", "lazy"):
        assert replay(roomy, mode, reserve=reserve).dump() == replay(roomy, mode).dump()


def test_reserve_zero_is_the_paper_model():
    """reserve = 0 (the default) is §5.5's on-demand eviction exactly."""
    for seed in range(5):
        t = tg.gen_c1(seed).slice_ops(0, 1500)
        for mode in ("base", "eager", "lazy"):
            assert replay(t, mode, reserve=0).dump() == replay(t, mode).dump()
