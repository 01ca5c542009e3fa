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
               device: int = 0, mem=None) -> um.Arena:
    return um.Arena(trace.block_bytes, trace.arena_bytes, trace.budget_bytes, flags=flags | mode_flags(mode),
                    host_pool_bytes=host_pool_bytes, device=device, mem=mem)


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


def issue(arena: um.Arena, trace, mode: str, start: int = 0, stop: int | None = None, stream=None) -> None:
    """Issue ops[start:stop] of the trace (no synchronization)."""
    a = arena.handle
    s = arena.stream_ptr if stream is None else stream
    ops, acc = trace.ops, trace.acc
    stop = len(ops) if stop is None else stop
    lazy = mode == "lazy"
    for r in ops[start:stop]:
        o = int(r["op"])
        if o == tg.OP_TOUCH:
            i, n = int(r["off"]), int(r["n"])
            um.um_touch_batch(a, acc[i:i + n], s)
        elif o == tg.OP_PREFETCH:
            um.um_prefetch(a, int(r["off"]), int(r["len"]), int(r["flags"]), s)
        elif o == tg.OP_DISCARD:
            if lazy and (int(r["flags"]) & tg.F_LAZY_OK):
                um.um_discard_lazy(a, int(r["off"]), int(r["len"]), s)
            else:
                um.um_discard(a, int(r["off"]), int(r["len"]), s)
        elif o == tg.OP_EVICT:
            um.um_evict(a, int(r["len"]), s)
        elif o == tg.OP_HOST_WRITE:
            um.um_host_write(a, int(r["off"]), int(r["len"]), s)
        else:
            raise ValueError(o)


def result(arena: um.Arena) -> dict:
    """The observable result (same keys as the oracle's dump())."""
    d = um.um_dump(arena.handle, arena.nblocks, arena.nframes)
    d["stats"] = um.um_get_stats(arena.handle)
    d["contents"] = um.um_content_tags(arena.handle, arena.nblocks)
    d["st"] = d["st"].astype(np.int64).tolist()
    return d


def run_trace(trace, mode: str, **kw) -> dict:
    arena = make_arena(trace, mode, **kw)
    try:
        alloc_buffers(arena, trace)
        issue(arena, trace, mode)
        return result(arena)
    finally:
        arena.close()
