"""Plain sequential simulator of the paper's UVM paging model with UvmDiscard /
UvmDiscardLazy — TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).

Every rule below cites PAPER.md (the text of Zhu et al., IISWC'22; "L<n>" = line n) or
the reading of SURVEY.md §8(c) ("A<n>") where the paper is silent; DESIGN.md lists the
readings.  Nothing here is blocked, fused or reordered: ops are applied one at a time,
blocks in ascending order, exactly as the transition table of SURVEY §8(c) states.

Per block b it tracks  st[b] in {U,H,HD,G,GE,GL},  key[b] (ukey while queued in USED,
dkey while queued in DISC),  gpu_stamp[b] / host_stamp[b] (content tags of the GPU frame
and of the host backing).  Frame ids are not part of the observable result, so only the
NUMBER of free frames is tracked.

States:
  U  never populated                      H  valid on host (Fig. 1 (1)/(3), L87)
  HD discarded, not on GPU (A5, L225)     G  valid, mapped, in USED (Fig. 1 (2), L87; L217)
  GE eager-discarded: unmapped, in DISC (§5.1; §5.5)
  GL lazy-discarded: mapped, SW dirty bit clear, in DISC (§5.2)
"""
from __future__ import annotations

U, H, HD, G, GE, GL = 0, 1, 2, 3, 4, 5
ST_NAMES = ("U", "H", "HD", "G", "GE", "GL")

STAT_NAMES = ("h2d_bytes", "d2h_bytes", "zf_bytes", "h2d_avoided_bytes", "d2h_avoided_bytes",
              "faults", "hits", "remaps", "unmaps", "revalidations", "refreshes", "evictions",
              "ops", "subops")

ACC_WRITE = 2


def stamp(seq: int, b: int) -> int:
    """Content tag written by the (simulated) application into block b during the
    (sub-)op numbered seq.  Non-zero because seq >= 1; tag 0 means "zero-filled"."""
    return (seq << 32) | b


class Oracle:
    """One arena: nblocks = arena_bytes / B virtual blocks, nframes = budget_bytes // B
    GPU frames (A15: oversubscription = arena / budget, L383)."""

    def __init__(self, block_bytes: int, arena_bytes: int, budget_bytes: int,
                 discard_off: bool = False, record: bool = False, host_release: bool = True,
                 overlap: int = 0, reserve: int = 0):
        if arena_bytes % block_bytes:
            raise ValueError("arena_bytes must be a multiple of block_bytes")
        self.B = block_bytes
        self.arena = arena_bytes
        self.nblocks = arena_bytes // block_bytes
        self.nframes = budget_bytes // block_bytes
        if self.nframes < 1:
            raise ValueError("budget smaller than one block")
        self.discard_off = discard_off          # "UVM-opt" baseline (§7.1)
        # host_release (reading R1 / SURVEY NEXT-4): a block's host copy exists
        # only while it is host-resident (H); it is released when the block migrates to
        # the GPU or is discarded.  The paper keeps CPU pages pinned (L87, L225); the only
        # observable difference is the stale value a discarded block reads back, and
        # §4.1 (L160) allows zeros there.  host_release=False is the paper-literal model.
        self.host_release = host_release
        # overlap (reading R7 / SURVEY NEXT-2): the application kernel of a
        # GPU sub-op may still run while the next sub-ops are serviced, as the paper's
        # asynchronous API calls overlap compute (L146, L166).  Victim selection then
        # also skips the blocks of the last `overlap` GPU sub-ops -- the longest suffix
        # of them that still leaves the current sub-op satisfiable (sizes summing with
        # |S| to at most nframes).  overlap = 0 is the sequential model of SURVEY §8(c).
        self.overlap = overlap
        # reserve (reading R12 / SURVEY NEXT-2, proactive eviction): the paper's
        # eviction process starts only "when the GPU's free page queue is empty" (§5.5
        # L219).  With reserve = R > 0 it also runs AHEAD of demand: after every GPU
        # sub-op with at least one block, if fewer than R frames are free, it reclaims
        # R - free more (best effort) in the same order (§5.5), skipping the
        # blocks of that sub-op and, with overlap, of every sub-op in the window (their
        # application kernels may still run).  Part of the sub-op: same seq, not an op.
        # Its write-backs can then overlap the application kernel (L146, L166, L381).
        self.reserve = reserve
        self.window: list = []                  # (blocks, count) of recent GPU sub-ops, oldest first
        n = self.nblocks
        self.st = [U] * n
        self.key = [0] * n
        self.gpu_stamp = [0] * n
        self.host_stamp = [0] * n               # host backing starts zeroed (Fig. 1 (1))
        # Page queues (§5.5).  Python dicts keep insertion order, and every
        # append happens in (seq, ascending block) order, so insertion order IS the
        # queue order: USED = pseudo-LRU, least recent first; DISC = FIFO.
        self.used: dict = {}
        self.disc: dict = {}
        self.free = self.nframes                # free page queue (L217)
        self.clock = 0
        self.stats = dict.fromkeys(STAT_NAMES, 0)
        self.log = [] if record else None       # (seq, "H2D"|"D2H"|"ZF", block, prev_state)

    # ------------------------------------------------------------------ helpers
    def _check(self, off: int, ln: int):
        if off < 0 or ln < 0 or off + ln > self.arena:
            raise ValueError("range outside the arena")     # UM_EINVAL, nothing applied

    def _cover(self, off: int, ln: int):
        """Blocks overlapping [off, off+len): touch/prefetch cover every overlapping
        block (§2.1: prefetch "pre-faults the virtual memory region")."""
        if ln == 0:
            return range(0)
        return range(off // self.B, (off + ln - 1) // self.B + 1)

    def _full(self, off: int, ln: int):
        """Blocks FULLY inside [off, off+len): discard "prefers full 2MB-aligned virtual
        regions and sometimes ignores partial ones" (§5.4) — A4: always ignore."""
        lo = -(-off // self.B)
        hi = (off + ln) // self.B
        return range(lo, max(lo, hi))

    def _next_seq(self) -> int:
        self.clock += 1
        self.stats["subops"] += 1
        return self.clock

    def _note(self, seq, kind, b, prev):
        if self.log is not None:
            self.log.append((seq, kind, b, prev))

    def _to_used(self, b: int, seq: int):
        """Transition into G: ukey = seq, append at the MRU end of USED ("Upon a GPU page
        fault or a prefetch operation, the underlying GPU physical pages are moved to the
        most recently used side of the queue", §5.5)."""
        self.st[b] = G
        self.key[b] = seq
        self.used[b] = seq

    def _select_victims(self, k: int, pinned) -> list:
        """Eviction order (§5.5): free queue first (handled by the caller via
        k = need - free), unused queue (empty, A12), then the discarded queue in FIFO
        order, then the LRU end of the used queue.  Blocks of the current sub-op are
        never victims (A3)."""
        out = []
        if k <= 0:
            return out
        for q in (self.disc, self.used):
            for b in q:
                if b not in pinned:
                    out.append(b)
                    if len(out) == k:
                        return out
        return out

    def _reclaim(self, v: int, seq: int):
        """Reclaim victim v's frame.  A valid page is swapped out to CPU DRAM (§5.3,
        §2.2; A10: every G victim is written back — no HW dirty bits, L174).  A
        discarded page is reclaimed without a transfer (§5.3, Fig. 2 (6) L131); a
        lazily discarded one needs its delayed unmap (§5.6)."""
        s = self.st[v]
        if s == G:
            self.host_stamp[v] = self.gpu_stamp[v]
            self.stats["d2h_bytes"] += self.B
            self._note(seq, "D2H", v, s)
            self.st[v] = H
            del self.used[v]
        elif s == GE:
            self.stats["d2h_avoided_bytes"] += self.B
            self.st[v] = HD
            del self.disc[v]
        elif s == GL:
            self.stats["d2h_avoided_bytes"] += self.B
            self.stats["unmaps"] += 1
            self.st[v] = HD
            del self.disc[v]
        else:  # pragma: no cover - queues only hold G/GE/GL blocks
            raise AssertionError("victim not GPU-resident")
        self.stats["evictions"] += 1
        self.free += 1

    # ------------------------------------------------------------------ GPU-destination sub-op
    def _gpu_subop(self, S: list, seq: int, touch: bool):
        """SURVEY §8(c) "Sub-op algorithm for a GPU-destination op", steps 1-7.
        S: ascending distinct blocks, len(S) <= nframes."""
        st = self.st
        pinned = set(S)
        if self.overlap:
            # R7: protect the blocks of the in-flight application kernels of the previous
            # GPU sub-ops; a window member is dropped (its kernel waited for) when keeping
            # it could leave fewer than k candidates
            keep, tot = [], len(S)
            for blocks, cnt in reversed(self.window[-self.overlap:]):
                if tot + cnt > self.nframes:
                    break
                tot += cnt
                keep.append(blocks)
            for blocks in keep:
                pinned |= blocks
            self.window = (self.window + [(frozenset(S), len(S))])[-self.overlap:]
        # steps 1-3: classify; blocks with no GPU frame need one
        need = [b for b in S if st[b] in (U, H, HD)]
        k = max(0, len(need) - self.free)
        # steps 4-5: choose and reclaim victims
        for v in self._select_victims(k, pinned):
            self._reclaim(v, seq)
        # steps 6-7, ascending block order (so USED appends are in (seq, block) order)
        sts = self.stats
        for b in S:
            s = st[b]
            if s in (U, H, HD):
                self.free -= 1
                if s == H:
                    # migrate touched data (§2.1; Fig. 1 (2) L87)
                    self.gpu_stamp[b] = self.host_stamp[b]
                    sts["h2d_bytes"] += self.B
                    self._note(seq, "H2D", b, s)
                    if self.host_release:
                        self.host_stamp[b] = 0
                else:
                    # never-touched -> zero-filled memory (§2.1); discarded and
                    # reclaimed -> "allocated, zero-filled, and mapped" instead of being
                    # migrated (§5.3, Fig. 2 (7) L131)
                    self.gpu_stamp[b] = 0
                    sts["zf_bytes"] += self.B
                    self._note(seq, "ZF", b, s)
                    if s == HD:
                        sts["h2d_avoided_bytes"] += self.B
                if touch:
                    sts["faults"] += 1
                self._to_used(b, seq)
            elif s == G:
                if touch:
                    sts["hits"] += 1        # A1: a resident access does not update recency
                else:
                    sts["refreshes"] += 1   # prefetch moves the page to MRU (L217)
                    del self.used[b]
                    self._to_used(b, seq)
            elif s == GE:
                # access after UvmDiscard, not yet reclaimed: "re-mapped and moved from the
                # discarded page queue to the most recently used side" (§5.7)
                sts["remaps"] += 1
                if touch:
                    sts["faults"] += 1      # unmapped => the access faults (§5.1)
                del self.disc[b]
                self._to_used(b, seq)
            else:  # GL
                if touch:
                    sts["hits"] += 1        # still mapped; A8: no notification, stays GL
                else:
                    # the mandatory prefetch sets the SW dirty bits (§5.2)
                    sts["revalidations"] += 1
                    del self.disc[b]
                    self._to_used(b, seq)

    def _evict_ahead(self, S: list, seq: int):
        """R12 proactive eviction after GPU sub-op `seq` over blocks S (see __init__)."""
        if self.reserve <= 0 or not S or self.free >= self.reserve:
            return
        pinned = set(S)
        if self.overlap:
            for blocks, _cnt in self.window:    # the last `overlap` GPU sub-ops, S included
                pinned |= blocks
        for v in self._select_victims(self.reserve - self.free, pinned):
            self._reclaim(v, seq)

    # ------------------------------------------------------------------ API ops
    def touch(self, accesses):
        """um_touch_batch: a batch of GPU accesses ("faults").  Distinct blocks are
        serviced in ascending sub-ops of <= nframes blocks (A3); after each sub-op the
        simulated application writes stamp(seq, b) into its WRITE blocks (step 8)."""
        for (off, ln, _k) in accesses:
            self._check(off, ln)
        blocks, writes = set(), set()
        for (off, ln, kind) in accesses:
            r = self._cover(off, ln)
            blocks.update(r)
            if kind & ACC_WRITE:
                writes.update(r)
        S = sorted(blocks)
        self.stats["ops"] += 1
        F = self.nframes
        chunks = [S[i:i + F] for i in range(0, len(S), F)] or [[]]
        for chunk in chunks:
            seq = self._next_seq()
            self._gpu_subop(chunk, seq, touch=True)
            for b in chunk:
                if b in writes:
                    self.gpu_stamp[b] = stamp(seq, b)   # a write after a discard is
                                                        # visible (§4.1)
            self._evict_ahead(chunk, seq)

    def prefetch(self, off: int, ln: int, dst: int):
        """um_prefetch (cudaMemPrefetchAsync, §2.1; Listing 2 L54-59)."""
        self._check(off, ln)
        if dst not in (0, 1):
            raise ValueError("bad dst")
        self.stats["ops"] += 1
        S = list(self._cover(off, ln))
        if dst == 0:
            F = self.nframes
            chunks = [S[i:i + F] for i in range(0, len(S), F)] or [[]]
            for chunk in chunks:
                seq = self._next_seq()
                self._gpu_subop(chunk, seq, touch=False)
                self._evict_ahead(chunk, seq)
            return
        seq = self._next_seq()
        st, sts = self.st, self.stats
        for b in S:
            s = st[b]
            if s == G:
                # migrate back to CPU pages (Fig. 1 (3), L87)
                self.host_stamp[b] = self.gpu_stamp[b]
                sts["d2h_bytes"] += self.B
                self._note(seq, "D2H", b, s)
                del self.used[b]
                self.free += 1
            elif s in (GE, GL):
                # discarded data needs no transfer (A9): the host keeps its old value,
                # which §4.1 L160 allows
                sts["d2h_avoided_bytes"] += self.B
                if s == GL:
                    sts["unmaps"] += 1
                del self.disc[b]
                self.free += 1
            st[b] = H   # U -> H (zero host page, Fig. 1 (1)); HD -> H (stale); H stays

    def discard(self, off: int, ln: int):
        """um_discard = UvmDiscard: eager unmap (§5.1).  G -> GE, moved from
        USED to the tail of DISC (§5.6, §5.5); GL -> GE keeps its DISC slot
        (A6); a host page stays pinned, H -> HD (§5.6, A5)."""
        self._check(off, ln)
        self.stats["ops"] += 1
        seq = self._next_seq()
        if self.discard_off:
            return          # UVM-opt baseline: accepted no-op that still consumes a seq (A18)
        st, sts = self.st, self.stats
        for b in self._full(off, ln):
            s = st[b]
            if s == G:
                del self.used[b]
                st[b] = GE
                self.key[b] = seq
                self.disc[b] = seq
                sts["unmaps"] += 1
            elif s == GL:
                st[b] = GE
                sts["unmaps"] += 1
            elif s == H:
                st[b] = HD
                if self.host_release:
                    self.host_stamp[b] = 0

    def discard_lazy(self, off: int, ln: int):
        """um_discard_lazy = UvmDiscardLazy: clear the software dirty bits, keep the
        mappings (§5.2).  G -> GL (into DISC); H -> HD."""
        self._check(off, ln)
        self.stats["ops"] += 1
        seq = self._next_seq()
        if self.discard_off:
            return
        st = self.st
        for b in self._full(off, ln):
            s = st[b]
            if s == G:
                del self.used[b]
                st[b] = GL
                self.key[b] = seq
                self.disc[b] = seq
            elif s == H:
                st[b] = HD
                if self.host_release:
                    self.host_stamp[b] = 0

    def evict(self, nbytes: int):
        """um_evict: make >= nbytes of frames free by the eviction policy (§5.5)."""
        if nbytes < 0:
            raise ValueError("bad size")
        self.stats["ops"] += 1
        seq = self._next_seq()
        want = -(-nbytes // self.B)
        for v in self._select_victims(want - self.free, ()):
            self._reclaim(v, seq)

    def free_range(self, off: int, ln: int):
        """um_free: the application releases [off, off+len) (cudaFree of managed memory).
        Reading R9: every FULLY covered block returns to U ("never
        populated", contents zero) with no transfer; a GPU frame it held goes to the
        unused page queue, which the eviction process reclaims before the discarded
        queue and without a transfer (§5.5) -- frames are anonymous, so it is
        counted with the free frames; a host copy is released."""
        self._check(off, ln)
        self.stats["ops"] += 1
        self._next_seq()
        for b in self._full(off, ln):
            s = self.st[b]
            if s == G:
                del self.used[b]
                self.free += 1
            elif s in (GE, GL):
                del self.disc[b]
                self.free += 1
            self.st[b] = U
            self.key[b] = 0
            self.gpu_stamp[b] = 0
            self.host_stamp[b] = 0

    def host_write(self, off: int, ln: int):
        """Harness op: the CPU writes new data into host-resident blocks ("Generate data,
        labels", Listing 6).  Requires every covered block to be in H."""
        self._check(off, ln)
        S = list(self._cover(off, ln))
        if any(self.st[b] != H for b in S):
            raise ValueError("host_write on a block that is not host-resident")
        self.stats["ops"] += 1
        seq = self._next_seq()
        for b in S:
            self.host_stamp[b] = stamp(seq, b)

    # ------------------------------------------------------------------ results
    def content(self, b: int) -> int:
        s = self.st[b]
        if s in (G, GE, GL):
            return self.gpu_stamp[b]
        if s in (H, HD):
            return self.host_stamp[b]
        return 0

    def contents(self) -> list:
        return [self.content(b) for b in range(self.nblocks)]

    def dump(self) -> dict:
        """The observable result compared bit-exactly with the CUDA path:
        per-block state, USED and DISC order, counters, content tags."""
        return {"st": list(self.st), "used_order": list(self.used), "disc_order": list(self.disc),
                "stats": dict(self.stats), "contents": self.contents(), "free": self.free}

    def check_conservation(self):
        """Invariant (vii): queues hold exactly the GPU-resident blocks and
        |G u GE u GL| + |free| = nframes."""
        g = [b for b, s in enumerate(self.st) if s == G]
        d = [b for b, s in enumerate(self.st) if s in (GE, GL)]
        assert sorted(self.used) == g, "USED != G blocks"
        assert sorted(self.disc) == d, "DISC != GE/GL blocks"
        assert len(g) + len(d) + self.free == self.nframes, "frame conservation"
        assert all(self.key[b] == k for b, k in self.used.items())
        assert all(self.key[b] == k for b, k in self.disc.items())
        for name in ("h2d_bytes", "d2h_bytes", "zf_bytes", "h2d_avoided_bytes", "d2h_avoided_bytes"):
            assert self.stats[name] % self.B == 0
        if self.host_release:   # R1: only host-resident blocks hold a host copy
            assert all(h == 0 for h, s in zip(self.host_stamp, self.st) if s != H)


MODES = ("base", "eager", "lazy")


def apply_op(o: Oracle, op: tuple, mode: str):
    """Apply one trace record (tracegen.Trace.iter_ops tuple) under a mode:
    base = UVM-opt (discards are no-ops), eager = every discard is UvmDiscard,
    lazy = lazy_ok discards become UvmDiscardLazy (§7.1; A17)."""
    kind, flags, off, ln, accs = op
    if kind == 0:
        o.touch(accs)
    elif kind == 1:
        o.prefetch(off, ln, flags)
    elif kind == 2:
        if mode == "lazy" and (flags & 1):
            o.discard_lazy(off, ln)
        else:
            o.discard(off, ln)
    elif kind == 3:
        o.evict(ln)
    elif kind == 4:
        o.host_write(off, ln)
    elif kind == 5:
        o.free_range(off, ln)
    else:
        raise ValueError(f"unknown op {kind}")


def replay(trace, mode: str = "eager", record: bool = False, stop: int | None = None,
           host_release: bool = True, overlap: int = 0, reserve: int = 0) -> Oracle:
    """Replay a tracegen.Trace (optionally only its first `stop` ops) in one mode."""
    if mode not in MODES:
        raise ValueError(mode)
    o = Oracle(trace.block_bytes, trace.arena_bytes, trace.budget_bytes,
               discard_off=(mode == "base"), record=record, host_release=host_release, overlap=overlap,
               reserve=reserve)
    for i, op in enumerate(trace.iter_ops()):
        if stop is not None and i >= stop:
            break
        apply_op(o, op, mode)
    return o
