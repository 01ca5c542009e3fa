"""Redundant memory transfer (RMT) accounting — TEST INFRASTRUCTURE ONLY (see
oracle/__init__.py).  SURVEY.md §8(c) item 7 ("rmt_analyze", M19), with reading R8 of
DESIGN.md.

The paper calls a transfer redundant when it moves data that is "overwritten before
being read" (§1); Fig. 3 (L125) sets the transfers an application requires against
those UVM performs, and Fig. 2 (L112, L131) shows the two it removes: the eviction
(D2H) of a dead buffer and its migration back (H2D) before it is overwritten.

This is an offline pass over a trace and a transfer log (the oracle's, or the CUDA
path's, which must be equal).  Data events of block b, in trace order:
  READ   a touch whose records covering b include UM_ACC_READ;
  WRITE  a touch whose records covering b include UM_ACC_WRITE (after its READ, if the
         touch also reads b: the application reads, then writes), or a host_write of b;
  DEAD   a discard (eager or lazy) that fully covers b (§5.4, A4), or a free of it.
Prefetch, evict and the paging layer's own moves are not data events.

A transfer (H2D or D2H) of b at op t moves b's value at that moment.  It is redundant iff
  (a) b's last WRITE or DEAD event before op t is DEAD — the value was already
      discarded (reads since then do not revive it), and a later read of it may return
      anything (§4.1)  [reading R8], or
  (b) b's first data event at or after op t is WRITE or DEAD — the value is overwritten
      or discarded before any read (L34).
The end of the trace counts as a read (final contents are checked), so a transfer with
no later data event is redundant only by (a).  Zero-fills move nothing over the link
and are not transfers.

SURVEY's wording of (b) alone would call the write-back of an already discarded block
"required" when nothing follows it; (a) is the reading that matches L34 + L160 (the
discarded value can never be legitimately read).  Both (a) and (b) are decided by the
trace alone, so the same transfer is judged the same way in every mode.
"""
from __future__ import annotations

from bisect import bisect_left

READ, WRITE, DEAD = 1, 2, 3
ACC_READ, ACC_WRITE = 1, 2
H2D, D2H, ZF = "H2D", "D2H", "ZF"
DISCARDED_STATES = (2, 4, 5)          # HD, GE, GL (oracle.sim numbering)


def _cover(B, off, ln):
    """Blocks overlapping [off, off+len) (touch, prefetch, host_write; §2.1)."""
    if ln == 0:
        return range(0)
    return range(off // B, (off + ln - 1) // B + 1)


def _full(B, off, ln):
    """Blocks fully inside [off, off+len) (discard; §5.4, A4)."""
    lo = -(-off // B)
    return range(lo, max(lo, (off + ln) // B))


def data_events(trace, unit=None):
    """Per block (per page of `unit` bytes at two levels): the ascending op indices of
    its data events and the events."""
    B = unit or trace.block_bytes
    idx, ev = {}, {}

    def add(b, t, e):
        idx.setdefault(b, []).append(t)
        ev.setdefault(b, []).append(e)

    for t, (kind, flags, off, ln, accs) in enumerate(trace.iter_ops()):
        if kind == 0:                                   # touch
            rd, wr = set(), set()
            for (o, n, k) in accs:
                r = _cover(B, o, n)
                if k & ACC_READ:
                    rd.update(r)
                if k & ACC_WRITE:
                    wr.update(r)
            for b in sorted(rd | wr):
                if b in rd:
                    add(b, t, READ)
                if b in wr:
                    add(b, t, WRITE)
        elif kind in (2, 5):                            # discard / discard_lazy / free
            for b in _full(B, off, ln):
                add(b, t, DEAD)
        elif kind == 4:                                 # host_write
            for b in _cover(B, off, ln):
                add(b, t, WRITE)
    return idx, ev


def op_seq_starts(trace):
    """First sequence number of every op (reading R2: one seq per op, one per sub-op of
    <= nframes distinct blocks for GPU-destination ops, at least one)."""
    B, F = trace.block_bytes, trace.budget_bytes // trace.block_bytes
    out, seq = [], 1
    for kind, flags, off, ln, accs in trace.iter_ops():
        out.append(seq)
        n = 1
        if kind == 0:
            blocks = set()
            for (o, m, _k) in accs:
                blocks.update(_cover(B, o, m))
            n = max(1, -(-len(blocks) // F))
        elif kind == 1 and flags == 0:                  # prefetch(GPU)
            n = max(1, -(-len(_cover(B, off, ln)) // F))
        seq += n
    return out


def log_by_op(trace, log):
    """Map a transfer log of (seq, kind, block, prev_state) to (op, kind, block, prev)."""
    starts = op_seq_starts(trace)
    return [(bisect_left(starts, s + 1) - 1, k, b, p) for (s, k, b, p) in log]


def redundant(idx, ev, t, b):
    """None if the move of b's value at op t is required, else the reason."""
    ti, te = idx.get(b, ()), ev.get(b, ())
    i = bisect_left(ti, t)
    j = i - 1
    while j >= 0 and te[j] == READ:
        j -= 1
    if j >= 0 and te[j] == DEAD:
        return "dead"                                   # (a)
    if i < len(ti) and te[i] in (WRITE, DEAD):
        return "overwritten" if te[i] == WRITE else "discarded"   # (b)
    return None


def rmt_analyze(trace, log, by_op=False, detail=False, page_bytes=None):
    """Redundant bytes of one run.  `log`: (seq, kind, block, prev_state) records (or
    (op, kind, block, prev_state) with by_op=True).  Returns byte totals, redundant
    bytes per direction and reason, and the moves of blocks that were in a discarded
    state (HD, GE, GL) when they moved — the north_star target is none in discard mode.
    detail=True adds the redundant records (op, kind, block, reason).  page_bytes: the
    log is per page (oracle.chunks); blocks in it are global page indices."""
    B = page_bytes or trace.block_bytes
    idx, ev = data_events(trace, B)
    recs = log if by_op else log_by_op(trace, log)
    out = {"h2d_bytes": 0, "d2h_bytes": 0, "rmt_h2d_bytes": 0, "rmt_d2h_bytes": 0,
           "reasons": {"dead": 0, "overwritten": 0, "discarded": 0}, "discarded_state_moves": 0}
    if detail:
        out["records"] = []
    for (t, kind, b, prev) in recs:
        if kind not in (H2D, D2H):
            continue
        out["h2d_bytes" if kind == H2D else "d2h_bytes"] += B
        if prev in DISCARDED_STATES:
            out["discarded_state_moves"] += 1
        r = redundant(idx, ev, t, b)
        if r:
            out["rmt_h2d_bytes" if kind == H2D else "rmt_d2h_bytes"] += B
            out["reasons"][r] += B
            if detail:
                out["records"].append((t, kind, b, r))
    out["rmt_bytes"] = out["rmt_h2d_bytes"] + out["rmt_d2h_bytes"]
    return out


def rmt_compare(base, disc):
    """RMT_base, RMT_left and avoided = (H2D+D2H)_base - (H2D+D2H)_discard (§8(c) item 7)."""
    tb = base["h2d_bytes"] + base["d2h_bytes"]
    td = disc["h2d_bytes"] + disc["d2h_bytes"]
    return {"rmt_base_bytes": base["rmt_bytes"], "rmt_left_bytes": disc["rmt_bytes"],
            "avoided_bytes": tb - td, "discarded_state_moves": disc["discarded_state_moves"]}
