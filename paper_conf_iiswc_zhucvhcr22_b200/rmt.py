"""Redundant-transfer report of a run: the library's transfer log (um_xlog_attach) judged
against the application's op stream (a tracegen.Trace) — measurement tooling of the
product, vectorised with numpy.  Never imports oracle/; tests/test_rmt_product.py pins it
record by record against the oracle's plain version (oracle/rmt.py).

Definition (PAPER §1: a transfer is redundant when its data is "overwritten before
being read"; Fig. 3; reading R8).  Data events of block b in op order:
READ (a touch reading b), WRITE (a touch writing b, after its read if it also reads; a
host_write), DEAD (a discard fully covering b, §5.4, or a free of it).  A move of b at op t is
redundant iff b's last WRITE-or-DEAD event before t is DEAD (the value was discarded,
§4.1), or b's first event at or after t is WRITE or DEAD.  The end of the trace
reads every block.
"""
from __future__ import annotations

import numpy as np

import tracegen as tg

EV_READ, EV_WRITE, EV_DEAD = 0, 1, 2     # order of events of one block within one op
_STATE_DISCARDED = (2, 4, 5)             # UM_ST_HD, UM_ST_GE, UM_ST_GL


def _expand(lo, hi):
    """Concatenated aranges [lo[i], hi[i]) and the index i of each element."""
    n = np.maximum(hi - lo, 0)
    tot = int(n.sum())
    if tot == 0:
        return np.zeros(0, np.int64), np.zeros(0, np.int64)
    rep = np.repeat(np.arange(len(lo)), n)
    start = np.repeat(np.cumsum(n) - n, n)
    return np.repeat(lo, n) + (np.arange(tot) - start), rep


def events(trace, unit=None):
    """Sorted event keys (block, op, order) packed in one int64, and the event kinds;
    blocks are units of `unit` bytes (pages at two levels), default the trace's block."""
    B = unit or trace.block_bytes
    ops = trace.ops
    T = len(ops) + 1
    blocks, times, kinds = [], [], []
    # touches: per access record, its covered blocks, READ / WRITE bits
    tidx = np.nonzero(ops["op"] == tg.OP_TOUCH)[0]
    if len(tidx):
        cnt = ops["n"][tidx].astype(np.int64)
        first = ops["off"][tidx].astype(np.int64)
        rec_op = np.repeat(tidx, cnt)
        rec = (np.repeat(first, cnt) + np.arange(int(cnt.sum())) - np.repeat(np.cumsum(cnt) - cnt, cnt))
        a = trace.acc[rec]
        ln = a["len"].astype(np.int64)
        keep = ln > 0
        off = a["off"].astype(np.int64)[keep]
        lo, hi = off // B, (off + ln[keep] - 1) // B + 1
        b, r = _expand(lo, hi)
        t = rec_op[keep][r]
        k = a["kind"][keep][r]
        # one READ and / or one WRITE per (block, op)
        for bit, ev in ((tg.ACC_READ, EV_READ), (tg.ACC_WRITE, EV_WRITE)):
            m = (k & bit) != 0
            key = np.unique(b[m] * T + t[m])
            blocks.append(key // T)
            times.append(key % T)
            kinds.append(np.full(len(key), ev, np.int64))
    for op, ev, full in ((tg.OP_DISCARD, EV_DEAD, True), (tg.OP_FREE, EV_DEAD, True), (tg.OP_HOST_WRITE, EV_WRITE, False)):
        idx = np.nonzero((ops["op"] == op) & (ops["len"] > 0))[0]
        off = ops["off"][idx].astype(np.int64)
        ln = ops["len"][idx].astype(np.int64)
        if full:
            lo, hi = -(-off // B), (off + ln) // B
        else:
            lo, hi = off // B, (off + ln - 1) // B + 1
        b, r = _expand(lo, hi)
        blocks.append(b)
        times.append(idx[r].astype(np.int64))
        kinds.append(np.full(len(b), ev, np.int64))
    b = np.concatenate(blocks) if blocks else np.zeros(0, np.int64)
    t = np.concatenate(times) if times else np.zeros(0, np.int64)
    k = np.concatenate(kinds) if kinds else np.zeros(0, np.int64)
    key = (b * T + t) * 3 + k
    o = np.argsort(key, kind="stable")
    return key[o], k[o], T


def op_of_seq(trace, seqs):
    """Op index of each sequence number (one seq per op; GPU-destination ops take one
    per sub-op of <= nframes distinct blocks, at least one: DESIGN.md R2)."""
    B, F = trace.block_bytes, trace.nframes
    per = np.ones(len(trace.ops), np.int64)
    for i, (kind, flags, off, ln, accs) in enumerate(trace.iter_ops()):
        if kind == tg.OP_TOUCH:
            iv = sorted((o // B, (o + m - 1) // B + 1) for (o, m, _k) in accs if m)
            n, hi = 0, -1
            for lo_, hi_ in iv:
                if lo_ >= hi:
                    n += hi_ - lo_
                    hi = hi_
                elif hi_ > hi:
                    n += hi_ - hi
                    hi = hi_
            per[i] = max(1, -(-n // F))
        elif kind == tg.OP_PREFETCH and flags == tg.DST_GPU and ln:
            per[i] = max(1, -(-((off + ln - 1) // B + 1 - off // B) // F))
    starts = np.cumsum(per) - per + 1
    return np.searchsorted(starts, np.asarray(seqs, np.int64), side="right") - 1


def analyze(trace, log, op_range=None, page_bytes=None):
    """log: (seq, kind, block, prev_state) records with kind in {"H2D", "D2H", "ZF"}, or
    an int array of rows (seq, block, kind 0/1/2, prev_state) as um_xlog records them.
    Returns byte totals, redundant bytes per direction, and the number of moves of
    blocks that were discarded (HD, GE, GL) when they moved.  op_range = (lo, hi) counts
    only the moves made by ops lo..hi-1 (e.g. one steady-state iteration).  page_bytes:
    a two-level arena's log (one record per page; blocks are global page indices)."""
    B = page_bytes or trace.block_bytes
    if len(log) and isinstance(log[0], tuple) and isinstance(log[0][1], str):
        code = {"H2D": 0, "D2H": 1, "ZF": 2}
        arr = np.array([(s, b, code[k], p) for (s, k, b, p) in log], np.int64).reshape(-1, 4)
    else:
        arr = np.asarray(log, np.int64).reshape(-1, 4)
    arr = arr[arr[:, 2] != 2]                       # zero-fills move nothing over the link
    t = op_of_seq(trace, arr[:, 0])
    if op_range is not None:
        m = (t >= op_range[0]) & (t < op_range[1])
        arr, t = arr[m], t[m]
    out = {"h2d_bytes": int((arr[:, 2] == 0).sum()) * B, "d2h_bytes": int((arr[:, 2] == 1).sum()) * B,
           "discarded_state_moves": int(np.isin(arr[:, 3], _STATE_DISCARDED).sum())}
    key, kind, T = events(trace, B)
    b = arr[:, 1]
    # last WRITE/DEAD event at or before each event index (per block), forward-filled
    wd = np.where(kind != EV_READ, np.arange(len(kind)), -1)
    last_wd = np.maximum.accumulate(wd) if len(wd) else wd
    i = np.searchsorted(key, (b * T + t) * 3, side="left")     # first event at/after (b, t)
    blk_of = key // (3 * T)
    prev_ok = i > 0
    j = np.where(prev_ok, last_wd[np.maximum(i - 1, 0)] if len(key) else -1, -1)
    dead = (j >= 0) & (blk_of[np.maximum(j, 0)] == b) & (kind[np.maximum(j, 0)] == EV_DEAD) if len(key) \
        else np.zeros(len(b), bool)
    nxt_ok = (i < len(key))
    ii = np.minimum(i, max(len(key) - 1, 0))
    over = nxt_ok & (blk_of[ii] == b) & (kind[ii] != EV_READ) if len(key) else np.zeros(len(b), bool)
    red = dead | over
    out["rmt_h2d_bytes"] = int((red & (arr[:, 2] == 0)).sum()) * B
    out["rmt_d2h_bytes"] = int((red & (arr[:, 2] == 1)).sum()) * B
    out["rmt_bytes"] = out["rmt_h2d_bytes"] + out["rmt_d2h_bytes"]
    return out
