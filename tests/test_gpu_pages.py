"""Two-level granularity on the CUDA path (include/um.h page_bytes):
2 MiB-style chunks of up to 32 pages, page-granular partial discards.  Parity with the
two-level oracle (oracle/chunks.py), bit-exact: chunk states, USED / DISC order, every
counter (bytes per page), per-page content tags, the dead / lazy page masks and the
per-page transfer log.  Run with `pytest -m gpu` on a B200."""
import numpy as np
import pytest

import tracegen as tg
from oracle.chunks import replay_chunks

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module", autouse=True)
def _cuda():
    torch = pytest.importorskip("torch")
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_iiswc_zhucvhcr22_b200 import build
    build.build()


def _xlog_cap(t, ppc):
    B, F = t.block_bytes, t.budget_bytes // t.block_bytes
    n = 0
    for kind, flags, off, ln, accs in t.iter_ops():
        if kind == tg.OP_TOUCH:
            n += 2 * sum((o + m - 1) // B - o // B + 1 for (o, m, _k) in accs if m)
        elif kind == tg.OP_PREFETCH:
            n += 2 * ((off + ln - 1) // B - off // B + 1 if ln else 0)
        elif kind == tg.OP_EVICT:
            n += min(F, ln // B + 1)
    return n * ppc + 64


def assert_page_parity(t, P, mode, **kw):
    from paper_conf_iiswc_zhucvhcr22_b200 import harness, um
    ppc = t.block_bytes // P
    o = replay_chunks(t, P, mode, record=True)
    d = o.dump()
    g = harness.run_trace(t, mode, page_bytes=P, flags=um.UM_F_APP_STAMP | um.UM_F_CHECK,
                          xlog=_xlog_cap(t, ppc), **kw)
    assert list(g["st"]) == d["st"]
    assert g["stats"] == d["stats"], {k: (g["stats"][k], d["stats"][k]) for k in d["stats"] if g["stats"][k] != d["stats"][k]}
    assert g["used_order"] == d["used_order"] and g["disc_order"] == d["disc_order"]
    assert g["dead"] == d["dead"] and g["lazy"] == d["lazy"]
    cg = np.asarray(g["contents"], np.uint64)
    co = np.asarray(d["contents"], np.uint64)
    bad = np.nonzero(cg != co)[0]
    assert len(bad) == 0, f"page contents differ at {bad[:8]}: gpu {[hex(x) for x in cg[bad[:4]]]} oracle {[hex(x) for x in co[bad[:4]]]}"
    assert g["xlog"] == sorted(o.log)
    return g, d


def _trace(P, ppc, nchunks, nframes, ops):
    C = P * ppc
    tb = tg.TraceBuilder(C, nchunks * C, nframes * C)
    for op in ops:
        kind = op[0]
        if kind == "touch":      # ("touch", [(first page, n pages, "R"|"W"|"RW")...])
            tb.touch([(q * P, n * P, {"R": tg.ACC_READ, "W": tg.ACC_WRITE, "RW": 3}[k]) for q, n, k in op[1]])
        elif kind == "discard":  # ("discard", first page, n pages, lazy)
            tb.discard(op[1] * P, op[2] * P, lazy_ok=op[3])
        elif kind == "prefetch":
            tb.prefetch(op[1] * P, op[2] * P, op[3])
        elif kind == "evict":
            tb.evict(op[1] * C)
        elif kind == "host_write":
            tb.host_write(op[1] * P, op[2] * P)
        elif kind == "free":     # ("free", first chunk, n chunks)
            tb.free(op[1] * C, op[2] * C)
        elif kind == "bytes":    # ("bytes", op, off, len[, extra]) raw byte ranges
            _, what, off, ln = op[:4]
            if what == "touch":
                tb.touch([(off, ln, op[4])])
            elif what == "discard":
                tb.discard(off, ln, lazy_ok=op[4])
            elif what == "prefetch":
                tb.prefetch(off, ln, op[4])
            elif what == "host_write":
                tb.host_write(off, ln)
    return tb.build()


P16 = 16 << 10


@pytest.mark.parametrize("mode", ["base", "eager", "lazy"])
def test_hand_scenarios(mode):
    """The hand-derived scenarios of tests/test_oracle_chunks.py at 16 KiB pages."""
    cases = [
        (2, 1, [("touch", [(0, 4, "W")]), ("discard", 0, 2, False), ("touch", [(4, 4, "W")]), ("touch", [(0, 4, "R")])]),
        (2, 1, [("touch", [(0, 4, "W")]), ("discard", 1, 2, True), ("touch", [(4, 4, "W")]),
                ("prefetch", 0, 4, tg.DST_GPU), ("touch", [(0, 4, "R")])]),
        (3, 2, [("prefetch", 0, 4, tg.DST_HOST), ("host_write", 0, 4), ("discard", 2, 2, False),
                ("touch", [(0, 2, "R")]), ("touch", [(4, 8, "W")]), ("prefetch", 0, 4, tg.DST_HOST)]),
        (2, 2, [("touch", [(0, 8, "W")]), ("bytes", "discard", 1000, 3 * P16 + 5000, False),
                ("evict", 2), ("touch", [(0, 8, "R")])]),
        (2, 1, [("touch", [(0, 8, "W")]), ("discard", 0, 4, False), ("discard", 4, 2, True),
                ("prefetch", 0, 8, tg.DST_HOST), ("touch", [(0, 8, "R")])]),
        (3, 2, [("touch", [(0, 8, "W")]), ("discard", 1, 2, False), ("free", 0, 1), ("touch", [(8, 4, "W")]),
                ("prefetch", 4, 4, tg.DST_HOST), ("free", 1, 1), ("touch", [(0, 4, "R")])]),
    ]
    for nchunks, nframes, ops in cases:
        assert_page_parity(_trace(P16, 4, nchunks, nframes, ops), P16, mode)


def _random_page_trace(seed, P, ppc, nchunks, nframes, n_ops=60):
    rng = np.random.default_rng(seed)
    npg = nchunks * ppc
    ops, host = [], False
    for _ in range(n_ops):
        r = rng.random()
        q = int(rng.integers(0, npg))
        n = int(rng.integers(1, min(2 * ppc, npg - q) + 1))
        if r < 0.42:
            recs = [(q, n, ["R", "W", "RW"][int(rng.integers(0, 3))])]
            if rng.random() < 0.3:
                q2 = int(rng.integers(0, npg))
                recs.append((q2, int(rng.integers(1, min(ppc, npg - q2) + 1)), "W"))
            ops.append(("touch", recs))
        elif r < 0.66:
            if rng.random() < 0.3:
                ops.append(("bytes", "discard", int(rng.integers(0, npg * P)), int(rng.integers(1, 3 * ppc * P)) // 1,
                            bool(rng.random() < 0.5)))
            else:
                ops.append(("discard", q, n, bool(rng.random() < 0.5)))
        elif r < 0.82:
            ops.append(("prefetch", q, n, tg.DST_GPU if rng.random() < 0.65 else tg.DST_HOST))
        elif r < 0.92:
            ops.append(("evict", int(rng.integers(1, nframes + 1))))
        else:
            # host_write needs host-resident chunks: prefetch them to the host first
            ops.append(("prefetch", q, n, tg.DST_HOST))
            ops.append(("host_write", q, n))
    # clip byte-range discards to the arena
    out = []
    for op in ops:
        if op[0] == "bytes":
            off = op[2]
            ln = min(op[3], npg * P - off)
            out.append(("bytes", op[1], off, ln, op[4]))
        else:
            out.append(op)
    return _trace(P, ppc, nchunks, nframes, out)


@pytest.mark.parametrize("seed", range(10))
@pytest.mark.parametrize("mode", ["base", "eager", "lazy"])
def test_random_16k_pages(seed, mode):
    rng = np.random.default_rng(1000 + seed)
    t = _random_page_trace(seed, P16, 4, int(rng.integers(2, 7)), int(rng.integers(1, 4)))
    assert_page_parity(t, P16, mode)


@pytest.mark.parametrize("seed", range(4))
@pytest.mark.parametrize("mode", ["eager", "lazy"])
def test_random_2m_chunks_64k_pages(seed, mode):
    """The paper's geometry: 2 MiB chunks of 32 pages of 64 KiB (L198, L209)."""
    rng = np.random.default_rng(2000 + seed)
    t = _random_page_trace(50 + seed, 64 << 10, 32, int(rng.integers(3, 8)), int(rng.integers(1, 4)), n_ops=80)
    assert_page_parity(t, 64 << 10, mode)


@pytest.mark.parametrize("mode", ["base", "eager", "lazy"])
def test_c3_two_level(mode):
    """C3 (Listing 6) at 2 MiB chunks with 64 KiB pages: buffer tails that a discard
    covers only in part become dead pages instead of being ignored (A4 at chunk level),
    so their write-back and migration are skipped too (the RMT_left of the single-level
    run, tests/test_rmt.py)."""
    t = tg.gen_c3(block_bytes=2 << 20, budget_bytes=384 << 20, iterations=2, workspace_bytes=5 << 20,
                  layers=tg.scale_layers(tg.VGG16, 1.0 / 64, 1.0 / 16), batch=6, discard_all_dead=True)
    assert t.arena_bytes > t.budget_bytes
    g, d = assert_page_parity(t, 64 << 10, mode)
    if mode != "base":
        assert any(d["dead"]) or d["stats"]["h2d_avoided_bytes"] > 0


def test_c3_two_level_removes_tail_rmt():
    """With pages, the discard-all-dead C3 run moves less redundant data: the chunk tails
    the single-level run kept moving are dead pages; only sub-page tails remain
    (tests/test_rmt_product.py pins the remainder to exactly those pages)."""
    from paper_conf_iiswc_zhucvhcr22_b200 import harness, rmt, um
    t = tg.gen_c3(block_bytes=2 << 20, budget_bytes=384 << 20, iterations=2, workspace_bytes=5 << 20,
                  layers=tg.scale_layers(tg.VGG16, 1.0 / 64, 1.0 / 16), batch=6, discard_all_dead=True)
    single = harness.run_trace(t, "eager", flags=um.UM_F_APP_STAMP, xlog=1 << 20)
    two = harness.run_trace(t, "eager", page_bytes=64 << 10, flags=um.UM_F_APP_STAMP, xlog=1 << 22)
    r1 = rmt.analyze(t, single["xlog"])
    r2 = rmt.analyze(t, two["xlog"], page_bytes=64 << 10)
    assert r1["rmt_bytes"] > 0 and r1["discarded_state_moves"] == 0
    assert r2["rmt_bytes"] < r1["rmt_bytes"] and r2["discarded_state_moves"] == 0
    assert r2["h2d_bytes"] + r2["d2h_bytes"] < r1["h2d_bytes"] + r1["d2h_bytes"]


def test_c3_full_size_two_level():
    """NEXT-1 at the bench's full size: C3 (discard-all-dead) at 1.5x of a ~170 GiB budget,
    2 MiB chunks of 64 KiB pages, two iterations; chunk states, queue orders, every counter,
    the page masks and every page's content tag (4.2 M pages) against oracle/chunks.py.
    (The per-page transfer log is compared at the smaller sizes above.)"""
    import gc
    import torch
    from paper_conf_iiswc_zhucvhcr22_b200 import harness, um
    gc.collect()
    torch.cuda.empty_cache()
    free, _ = torch.cuda.mem_get_info()
    GiB = 1 << 30
    budget = min(170 * GiB, free - 8 * GiB) // (2 << 20) * (2 << 20)
    assert budget >= 160 * GiB, f"only {free / GiB:.1f} GiB free"
    t = tg.gen_c3(block_bytes=2 << 20, budget_bytes=budget, oversub=1.5, iterations=2, discard_all_dead=True)
    P = 64 << 10
    pool = t.arena_bytes - t.budget_bytes + (2 << 30)
    g = harness.run_trace(t, "eager", page_bytes=P, flags=um.UM_F_APP_STAMP | um.UM_F_CHECK, host_pool_bytes=pool)
    d = replay_chunks(t, P, "eager").dump()
    assert list(g["st"]) == d["st"]
    assert g["stats"] == d["stats"], {k: (g["stats"][k], d["stats"][k]) for k in d["stats"] if g["stats"][k] != d["stats"][k]}
    assert g["used_order"] == d["used_order"] and g["disc_order"] == d["disc_order"]
    assert g["dead"] == d["dead"] and g["lazy"] == d["lazy"]
    assert any(d["dead"])
    cg = np.asarray(g["contents"], np.uint64)
    co = np.asarray(d["contents"], np.uint64)
    bad = np.nonzero(cg != co)[0]
    assert len(bad) == 0, f"page contents differ at {bad[:8]}"
