"""Replay a tracegen.Trace through libum (the CUDA path) — harness, not the product.

Mode mapping (§7.1): base = UVM-opt (arena flag UM_F_DISCARD_OFF: discards
are accepted no-ops), eager = every discard is um_discard, lazy = discards marked
lazy_ok become um_discard_lazy.  Never imports oracle/.
"""
from __future__ import annotations

import numpy as np

import tracegen as tg
from . import um


def mode_flags(mode: str) -> int:
    if mode not in ("base", "eager", "lazy"):
        raise ValueError(mode)
    return um.UM_F_DISCARD_OFF if mode == "base" else 0


def make_arena(trace, mode: str, *, flags: int = um.UM_F_APP_STAMP | um.UM_F_CHECK, host_pool_bytes=None,
               device: int | None = None, mem=None, page_bytes: int = 0, reserve_blocks: int = 0) -> um.Arena:
    """page_bytes < block_bytes: a two-level arena (chunks of block_bytes, pages of
    page_bytes).  reserve_blocks > 0: proactive eviction (R12)."""
    return um.Arena(trace.block_bytes, trace.arena_bytes, trace.budget_bytes, flags=flags | mode_flags(mode),
                    host_pool_bytes=host_pool_bytes, device=device, mem=mem, page_bytes=page_bytes,
                    reserve_blocks=reserve_blocks)


def alloc_buffers(arena: um.Arena, trace) -> None:
    for name, (off, nbytes) in trace.buffers.items():
        got = um.um_alloc(arena.handle, nbytes)
        if got != off:
            raise AssertionError(f"um_alloc({name}) = {got}, trace expects {off}")


def iteration_bounds(trace) -> list:
    """Op index ranges of the iterations of a periodic trace (C3)."""
    it = int(trace.meta.get("iterations", 1))
    per = len(trace.ops) // it
    return [(i * per, (i + 1) * per) for i in range(it)]


def _dev_records(trace, device: int | None = None) -> int:
    """The trace's access records copied once into device memory (the GPU's fault buffer
    analogue for um_touch_batch_dev); returns its device address."""
    import torch
    if device is None:
        device = torch.cuda.current_device()
    key = f"_acc_dev{device}"
    t = trace.meta.get(key)
    if t is None:
        acc = np.ascontiguousarray(trace.acc).view(np.uint8).reshape(-1)
        t = torch.empty(max(16, acc.size), dtype=torch.uint8, device=torch.device("cuda", device))
        if acc.size:
            t[:acc.size].copy_(torch.from_numpy(acc))
        torch.cuda.synchronize(device)   # the arena's streams do not wait for torch's
        trace.meta[key] = t
    return t.data_ptr()


def _calls(trace, mode: str, dev_records: bool = False) -> list:
    """The trace as a list of (libum function, args-after-arena) tuples, built once per
    (trace, mode): the issue loop then only makes the ctypes calls.  dev_records: touch
    batches go through um_touch_batch_dev with the records in device memory."""
    key = "_calls_" + mode + ("_dev" if dev_records else "")
    cached = trace.meta.get(key)
    if cached is not None:
        return cached
    L = um.lib()
    acc = np.ascontiguousarray(trace.acc)
    trace.meta["_acc_keepalive"] = acc
    base = acc.ctypes.data
    dbase = _dev_records(trace) if dev_records else 0
    lazy = mode == "lazy"
    out = []
    for r in trace.ops.tolist():          # (op, flags, n, off, len) as python ints
        o, fl, n, off, ln = r
        if o == tg.OP_TOUCH and dev_records:
            out.append(("um_touch_batch_dev", L.um_touch_batch_dev, (dbase + 16 * off if n else None, n)))
        elif o == tg.OP_TOUCH:
            out.append(("um_touch_batch", L.um_touch_batch, (base + 16 * off if n else None, n)))
        elif o == tg.OP_PREFETCH:
            out.append(("um_prefetch", L.um_prefetch, (off, ln, fl)))
        elif o == tg.OP_DISCARD:
            if lazy and (fl & tg.F_LAZY_OK):
                out.append(("um_discard_lazy", L.um_discard_lazy, (off, ln)))
            else:
                out.append(("um_discard", L.um_discard, (off, ln)))
        elif o == tg.OP_EVICT:
            out.append(("um_evict", L.um_evict, (ln,)))
        elif o == tg.OP_HOST_WRITE:
            out.append(("um_host_write", L.um_host_write, (off, ln)))
        elif o == tg.OP_FREE:
            out.append(("um_free", L.um_free, (off, ln)))
        else:
            raise ValueError(o)
    trace.meta[key] = out
    return out


def issue(arena: um.Arena, trace, mode: str, start: int = 0, stop: int | None = None, stream=None,
          dev_records: bool = False) -> None:
    """Issue ops[start:stop] of the trace through the C ABI (no synchronization)."""
    a = arena.handle
    s = arena.stream_ptr if stream is None else stream
    calls = _calls(trace, mode, dev_records)
    stop = len(calls) if stop is None else stop
    for name, fn, args in calls[start:stop]:
        st = fn(a, *args, s)
        if st:
            raise um.UmError(name, st)


def result(arena: um.Arena) -> dict:
    """The observable result (same keys as the oracle's dump())."""
    d = um.um_dump(arena.handle, arena.nblocks, arena.nframes)
    d["stats"] = um.um_get_stats(arena.handle)
    d["contents"] = um.um_content_tags(arena.handle, arena.nblocks * arena.ppc)
    d["st"] = d["st"].astype(np.int64).tolist()
    if arena.ppc > 1:
        dead, lazy = um.um_page_masks(arena.handle, arena.nblocks)
        d["dead"], d["lazy"] = dead.astype(np.int64).tolist(), lazy.astype(np.int64).tolist()
    return d


class XLog:
    """A device buffer attached as the arena's transfer log (um_xlog_attach)."""

    def __init__(self, arena: um.Arena, cap: int):
        import torch
        self.arena, self.cap = arena, cap
        # torch allocates on its current stream; the arena's paging stream does not wait for
        # it, so the buffer is handed over only once torch's work on it is done (no zeroing:
        # only the records appended are read)
        self.buf = torch.empty((cap, 4), dtype=torch.int32, device=arena.frames.device)
        torch.cuda.synchronize(arena.frames.device)
        um.um_xlog_attach(arena.handle, self.buf.data_ptr(), cap)

    def raw(self) -> np.ndarray:
        """The records as an int64 array of rows (seq, block, kind, prev_state)."""
        n = um.um_xlog_count(self.arena.handle)
        if n > self.cap:
            raise RuntimeError(f"transfer log overflow: {n} records > capacity {self.cap}")
        return self.buf[:n].cpu().numpy().view(np.uint32).astype(np.int64)

    def records(self) -> list:
        """(seq, kind, block, prev_state) tuples, sorted (the log's order is arbitrary)."""
        n = um.um_xlog_count(self.arena.handle)
        if n > self.cap:
            raise RuntimeError(f"transfer log overflow: {n} records > capacity {self.cap}")
        a = self.buf[:n].cpu().numpy().view(np.uint32).astype(np.int64)
        return sorted((int(s), um.XL_KIND[k], int(b), int(p)) for s, b, k, p in a.tolist())

    def detach(self):
        um.um_xlog_attach(self.arena.handle, None, 0)


def run_trace(trace, mode: str, xlog: int = 0, dev_records: bool = False, **kw) -> dict:
    """Replay the whole trace on a fresh arena; xlog = capacity of a transfer log to
    attach (its sorted records are returned under "xlog"); dev_records: touch batches
    from device memory (um_touch_batch_dev)."""
    arena = make_arena(trace, mode, **kw)
    try:
        alloc_buffers(arena, trace)
        lg = XLog(arena, xlog) if xlog else None
        issue(arena, trace, mode, dev_records=dev_records)
        r = result(arena)
        if lg:
            r["xlog"] = lg.records()
            lg.detach()
        return r
    finally:
        arena.close()
