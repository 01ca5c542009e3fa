"""Two-level granularity — TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).

A plain sequential CPU model of 2 MiB chunks holding 64 KiB pages, written step by step
from the paper and DESIGN.md §12 (proposed reading, pinned here before any kernel):

  * the chunk stays the residency and eviction unit: "allocate, zero, and map a 2MB
    physical page upon first touch" (§5.4), "swapping out a 2MB GPU physical page"
    (§5.3), page queues hold chunks (§5.5).  Every chunk-level rule of
    oracle.sim (states U H HD G GE GL, USED / DISC order, victims, A1-A18) is unchanged;
  * a discard that covers whole chunks acts at chunk level exactly as in oracle.sim;
  * a discard that covers only some pages of a chunk marks them *dead* without
    unmapping or re-queueing the chunk ("avoid splitting 2MB GPU mappings from partial
    unmapping requests", §5.4).  Pages partially covered are ignored (A4);
  * "the UVM system will skip the memory transfers of the underlying physical page until
    it gets accessed again" (§5.3): evicting (or prefetching to the host) a chunk
    writes back only its live pages; migrating a chunk to the GPU zero-fills its dead
    pages instead of migrating them (L200);
  * "accessed again": a touch revives the eagerly discarded pages it covers; a lazily
    discarded page (UvmDiscardLazy) is revived only by a prefetch, either destination
    (§5.2, A8, A17); a host_write revives the pages it writes;
  * the prepared bit (§5.7) stays implied (A14): every page of a GPU-resident chunk
    has been zero-filled or migrated.

Per chunk c: the chunk state of oracle.sim plus `dead[c]` (pages discarded and not
accessed since) and `lazy[c]` (the subset discarded lazily), bit p = page p of the
chunk; both are 0 in the chunk-level discarded states.  Contents are tracked per page:
stamp(seq, global page index).  Byte counters count pages moved / avoided; event
counters (faults, hits, evictions, ...) count chunks as in oracle.sim.

Parity status: pinned by hand-derived scenarios and the reduction to oracle.sim when
every discard is chunk-aligned (tests/test_oracle_chunks.py); no CUDA path yet.
"""
from __future__ import annotations

from .sim import ACC_WRITE, G, GE, GL, H, HD, U, Oracle, stamp


class ChunkOracle(Oracle):
    """One arena of chunks of `block_bytes` split into pages of `page_bytes`."""

    def __init__(self, block_bytes: int, page_bytes: int, arena_bytes: int, budget_bytes: int,
                 discard_off: bool = False, record: bool = False, host_release: bool = True):
        if block_bytes % page_bytes or not 1 <= block_bytes // page_bytes <= 32:
            raise ValueError("a chunk holds 1..32 whole pages")
        super().__init__(block_bytes, arena_bytes, budget_bytes, discard_off=discard_off, record=record,
                         host_release=host_release)
        self.P = page_bytes
        self.ppc = block_bytes // page_bytes
        n = self.nblocks
        self.dead = [0] * n
        self.lazy = [0] * n
        self.gpu_ps = [0] * (n * self.ppc)      # per-page content of the GPU frame
        self.host_ps = [0] * (n * self.ppc)     # per-page content of the host backing

    # ------------------------------------------------------------------ page helpers
    def _pages_cover(self, off: int, ln: int):
        """Pages overlapping [off, off+len) (touch, prefetch, host_write)."""
        if ln == 0:
            return range(0)
        return range(off // self.P, (off + ln - 1) // self.P + 1)

    def _pages_full(self, off: int, ln: int):
        """Pages fully inside [off, off+len) (discard, A4 at page granularity)."""
        lo = -(-off // self.P)
        return range(lo, max(lo, (off + ln) // self.P))

    def _by_chunk(self, pages) -> dict:
        """{chunk: page bit mask} of a set of global page indices."""
        out: dict = {}
        for q in pages:
            c, p = divmod(q, self.ppc)
            out[c] = out.get(c, 0) | (1 << p)
        return out

    # ------------------------------------------------------------------ data movement
    def _reclaim(self, v: int, seq: int):
        """Victim v leaves the GPU.  A valid chunk (G) writes back its live pages only;
        its dead pages need no transfer (§5.3) and stay dead on the host."""
        if self.st[v] != G:
            return super()._reclaim(v, seq)          # GE / GL: chunk-level, no transfer
        self._chunk_to_host(v, seq)
        self.st[v] = H
        del self.used[v]
        self.stats["evictions"] += 1
        self.free += 1

    def _chunk_to_host(self, c: int, seq: int):
        P, base = self.P, c * self.ppc
        for p in range(self.ppc):
            if (self.dead[c] >> p) & 1:
                self.stats["d2h_avoided_bytes"] += P
                if self.host_release:
                    self.host_ps[base + p] = 0
            else:
                self.host_ps[base + p] = self.gpu_ps[base + p]
                self.stats["d2h_bytes"] += P
                self._note(seq, "D2H", base + p, G)

    def _chunk_to_gpu(self, c: int, s: int, seq: int):
        """Chunk c (state s in U/H/HD) gets a frame.  U and HD chunks are zero-filled
        whole (L76, L200); an H chunk migrates its live pages and zero-fills its dead
        ones (L200)."""
        P, base = self.P, c * self.ppc
        for p in range(self.ppc):
            q = base + p
            if s == H and not (self.dead[c] >> p) & 1:
                self.gpu_ps[q] = self.host_ps[q]
                self.stats["h2d_bytes"] += P
                self._note(seq, "H2D", q, s)
            else:
                self.gpu_ps[q] = 0
                self.stats["zf_bytes"] += P
                self._note(seq, "ZF", q, s)
                if s == HD or (s == H and (self.dead[c] >> p) & 1):
                    self.stats["h2d_avoided_bytes"] += P
            if s == H and self.host_release:
                self.host_ps[q] = 0

    # ------------------------------------------------------------------ GPU-destination sub-op
    def _gpu_subop(self, S: list, seq: int, touch: bool):
        """oracle.sim's sub-op steps 1-7 with page-granular data movement."""
        st = self.st
        pinned = set(S)
        need = [b for b in S if st[b] in (U, H, HD)]
        k = max(0, len(need) - self.free)
        for v in self._select_victims(k, pinned):
            self._reclaim(v, seq)
        sts = self.stats
        for b in S:
            s = st[b]
            if s in (U, H, HD):
                self.free -= 1
                self._chunk_to_gpu(b, s, seq)
                if s != H:
                    self.dead[b] = self.lazy[b] = 0
                if touch:
                    sts["faults"] += 1
                self._to_used(b, seq)
            elif s == G:
                if touch:
                    sts["hits"] += 1
                else:
                    sts["refreshes"] += 1
                    del self.used[b]
                    self._to_used(b, seq)
            elif s == GE:
                sts["remaps"] += 1
                if touch:
                    sts["faults"] += 1
                del self.disc[b]
                self._to_used(b, seq)
            else:  # GL
                if touch:
                    sts["hits"] += 1
                else:
                    sts["revalidations"] += 1
                    del self.disc[b]
                    self._to_used(b, seq)

    # ------------------------------------------------------------------ API ops
    def touch(self, accesses):
        for (off, ln, _k) in accesses:
            self._check(off, ln)
        pages, writes = set(), set()
        for (off, ln, kind) in accesses:
            r = self._pages_cover(off, ln)
            pages.update(r)
            if kind & ACC_WRITE:
                writes.update(r)
        cover = self._by_chunk(pages)
        S = sorted(cover)
        self.stats["ops"] += 1
        F = self.nframes
        for chunk in [S[i:i + F] for i in range(0, len(S), F)] or [[]]:
            seq = self._next_seq()
            self._gpu_subop(chunk, seq, touch=True)
            for c in chunk:
                # accessed again: eagerly discarded pages revive, lazy ones do not (A8)
                self.dead[c] &= ~(cover[c] & ~self.lazy[c])
                for p in range(self.ppc):
                    q = c * self.ppc + p
                    if q in writes:
                        self.gpu_ps[q] = stamp(seq, q)

    def prefetch(self, off: int, ln: int, dst: int):
        self._check(off, ln)
        if dst not in (0, 1):
            raise ValueError("bad dst")
        self.stats["ops"] += 1
        cover = self._by_chunk(self._pages_cover(off, ln))
        S = sorted(cover)
        if dst == 0:
            F = self.nframes
            for chunk in [S[i:i + F] for i in range(0, len(S), F)] or [[]]:
                self._gpu_subop(chunk, self._next_seq(), touch=False)
        else:
            seq = self._next_seq()
            st, sts = self.st, self.stats
            for c in S:
                s = st[c]
                if s == G:
                    self._chunk_to_host(c, seq)
                    del self.used[c]
                    self.free += 1
                elif s in (GE, GL):
                    sts["d2h_avoided_bytes"] += self.B
                    if s == GL:
                        sts["unmaps"] += 1
                    del self.disc[c]
                    self.free += 1
                st[c] = H
        # a prefetch to either destination revalidates the pages it covers (A17)
        for c, m in cover.items():
            self.dead[c] &= ~m
            self.lazy[c] &= ~m

    def _partial(self, off: int, ln: int, lazy: bool):
        """Pages of chunks the range covers only in part (chunk in G or H)."""
        full = set(self._full(off, ln))
        for c, m in self._by_chunk(self._pages_full(off, ln)).items():
            if c in full or self.st[c] not in (G, H):
                continue
            if lazy:
                self.lazy[c] |= m & ~self.dead[c]
            else:
                self.lazy[c] &= ~m
            self.dead[c] |= m
            if self.st[c] == H and self.host_release:   # R1: host copy released
                for p in range(self.ppc):
                    if (m >> p) & 1:
                        self.host_ps[c * self.ppc + p] = 0

    def _chunk_level(self, off: int, ln: int):
        for c in self._full(off, ln):
            self.dead[c] = self.lazy[c] = 0

    def discard(self, off: int, ln: int):
        st0 = list(self.st) if not self.discard_off else None
        super().discard(off, ln)
        if self.discard_off:
            return
        for c in self._full(off, ln):
            if st0[c] == H and self.host_release:
                for p in range(self.ppc):
                    self.host_ps[c * self.ppc + p] = 0
        self._chunk_level(off, ln)
        self._partial(off, ln, lazy=False)

    def discard_lazy(self, off: int, ln: int):
        st0 = list(self.st) if not self.discard_off else None
        super().discard_lazy(off, ln)
        if self.discard_off:
            return
        for c in self._full(off, ln):
            if st0[c] == H and self.host_release:
                for p in range(self.ppc):
                    self.host_ps[c * self.ppc + p] = 0
        self._chunk_level(off, ln)
        self._partial(off, ln, lazy=True)

    def free_range(self, off: int, ln: int):
        """um_free (R9) at chunk level: fully covered chunks return to U, page state with them."""
        super().free_range(off, ln)
        for c in self._full(off, ln):
            self.dead[c] = self.lazy[c] = 0
            for p in range(self.ppc):
                self.gpu_ps[c * self.ppc + p] = self.host_ps[c * self.ppc + p] = 0

    def host_write(self, off: int, ln: int):
        self._check(off, ln)
        cover = self._by_chunk(self._pages_cover(off, ln))
        if any(self.st[c] != H for c in cover):
            raise ValueError("host_write on a chunk that is not host-resident")
        self.stats["ops"] += 1
        seq = self._next_seq()
        for c, m in cover.items():
            self.dead[c] &= ~m
            self.lazy[c] &= ~m
            for p in range(self.ppc):
                if (m >> p) & 1:
                    self.host_ps[c * self.ppc + p] = stamp(seq, c * self.ppc + p)

    # ------------------------------------------------------------------ results
    def content(self, q: int) -> int:
        """Content tag of global page q."""
        s = self.st[q // self.ppc]
        if s in (G, GE, GL):
            return self.gpu_ps[q]
        if s in (H, HD):
            return self.host_ps[q]
        return 0

    def contents(self) -> list:
        return [self.content(q) for q in range(self.nblocks * self.ppc)]

    def dump(self) -> dict:
        d = super().dump()
        d["dead"], d["lazy"] = list(self.dead), list(self.lazy)
        return d

    def check_conservation(self):
        """oracle.sim's invariant (vii) at chunk level, byte counters in pages, masks only
        where the chunk itself is not discarded."""
        g = [b for b, s in enumerate(self.st) if s == G]
        d = [b for b, s in enumerate(self.st) if s in (GE, GL)]
        assert sorted(self.used) == g, "USED != G chunks"
        assert sorted(self.disc) == d, "DISC != GE/GL chunks"
        assert len(g) + len(d) + self.free == self.nframes, "frame conservation"
        if self.host_release:
            for q, h in enumerate(self.host_ps):
                assert h == 0 or self.st[q // self.ppc] == H, "host copy only while host-resident"
        for name in ("h2d_bytes", "d2h_bytes", "zf_bytes", "h2d_avoided_bytes", "d2h_avoided_bytes"):
            assert self.stats[name] % self.P == 0
        for c, s in enumerate(self.st):
            assert self.lazy[c] & ~self.dead[c] == 0, "lazy pages are dead pages"
            if s not in (G, H):
                assert self.dead[c] == 0, "page masks only in G / H"


def replay_chunks(trace, page_bytes: int, mode: str = "eager", record: bool = False,
                  host_release: bool = True) -> ChunkOracle:
    """Replay a tracegen.Trace (block_bytes = chunk bytes) with pages of page_bytes."""
    from .sim import MODES, apply_op
    if mode not in MODES:
        raise ValueError(mode)
    o = ChunkOracle(trace.block_bytes, page_bytes, trace.arena_bytes, trace.budget_bytes,
                    discard_off=(mode == "base"), record=record, host_release=host_release)
    for op in trace.iter_ops():
        apply_op(o, op, mode)
    return o
