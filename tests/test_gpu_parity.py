"""Parity of the CUDA path (libum.so, called through the C ABI) with the CPU oracle:
per-block final state, USED/DISC order, every counter and every block's content tag
must match bit-exactly.  Run with `pytest -m gpu` on a B200."""
import os

import numpy as np
import pytest

import tracegen as tg
from oracle.sim import replay as oracle_replay
import scenarios as scn

pytestmark = pytest.mark.gpu

SCEN = scn.load()


@pytest.fixture(scope="module", autouse=True)
def _cuda():
    torch = pytest.importorskip("torch")
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_iiswc_zhucvhcr22_b200 import build
    build.build()


COPY_FLAGS = {"default": 0, "kernel": 32, "ce": 2}   # default = the TMA kernel K4; UM_F_COPY_KERNEL / UM_F_COPY_CE


def xlog_bound(trace, reserve=0):
    """Upper bound on the transfer-log records of a trace: every covered block of a GPU
    op may bring one newcomer record and one victim write-back, every block of a
    prefetch(HOST) or evict one write-back; with proactive eviction (R12) every GPU
    sub-op may add `reserve` write-backs."""
    B, F = trace.block_bytes, trace.budget_bytes // trace.block_bytes
    n = 0
    for kind, flags, off, ln, accs in trace.iter_ops():
        if kind == tg.OP_TOUCH:
            nb = sum((o + m - 1) // B - o // B + 1 for (o, m, _k) in accs if m)
            n += 2 * nb + reserve * (nb // F + 1)
        elif kind == tg.OP_PREFETCH:
            nb = (off + ln - 1) // B - off // B + 1 if ln else 0
            n += (2 if flags == tg.DST_GPU else 1) * nb + (reserve * (nb // F + 1) if flags == tg.DST_GPU else 0)
        elif kind == tg.OP_EVICT:
            n += min(F, ln // B + 1)
    return n + 64


def _gpu(trace, mode, copy="default", overlap=False, xlog=True, reserve=0, **kw):
    """The CUDA path's result, with the transfer log attached (xlog_bound capacity)."""
    from paper_conf_iiswc_zhucvhcr22_b200 import harness, um
    flags = um.UM_F_APP_STAMP | um.UM_F_CHECK | COPY_FLAGS[copy] | (um.UM_F_OVERLAP if overlap else 0)
    if reserve:
        kw["reserve_blocks"] = reserve
    return harness.run_trace(trace, mode, flags=flags, xlog=xlog_bound(trace, reserve) if xlog else 0, **kw)


OVERLAP_W = 2   # kOverlapW in csrc/um_internal.h (reading R7)


def _first_diff(a, b):
    for i, (x, y) in enumerate(zip(a, b)):
        if x != y:
            return f"transfer log differs at record {i}: gpu {x} oracle {y} (lengths {len(a)}, {len(b)})"
    return f"transfer log lengths differ: gpu {len(a)} oracle {len(b)}"


def assert_parity(trace, mode, g=None, overlap=False, reserve=0):
    g = g if g is not None else _gpu(trace, mode, overlap=overlap, reserve=reserve)
    orc = oracle_replay(trace, mode, overlap=OVERLAP_W if overlap else 0, record="xlog" in g, reserve=reserve)
    o = orc.dump()
    if "xlog" in g:
        # every H2D / D2H / zero-fill, with its sub-op seq and the block's prior state
        assert g["xlog"] == sorted(orc.log), _first_diff(g["xlog"], sorted(orc.log))
    st_g = np.asarray(g["st"])
    st_o = np.asarray(o["st"])
    bad = np.nonzero(st_g != st_o)[0]
    assert len(bad) == 0, f"state mismatch at blocks {bad[:10]}: gpu {st_g[bad[:10]]} oracle {st_o[bad[:10]]}"
    assert g["stats"] == o["stats"], {k: (g["stats"][k], o["stats"][k]) for k in o["stats"] if g["stats"][k] != o["stats"][k]}
    assert g["used_order"] == o["used_order"]
    assert g["disc_order"] == o["disc_order"]
    ct_g = np.asarray(g["contents"], dtype=np.uint64)
    ct_o = np.asarray(o["contents"], dtype=np.uint64)
    badc = np.nonzero(ct_g != ct_o)[0]
    assert len(badc) == 0, f"content mismatch at {badc[:10]}: gpu {[hex(x) for x in ct_g[badc[:5]]]} oracle {[hex(x) for x in ct_o[badc[:5]]]}"
    return g, o


@pytest.mark.parametrize("name", sorted(SCEN))
def test_scenarios(name):
    sc = SCEN[name]
    trace, mode = scn.build(sc)
    ov = sc.get("overlap", 0)
    assert ov in (0, OVERLAP_W)
    g, _ = assert_parity(trace, mode, overlap=bool(ov), reserve=sc.get("reserve", 0))
    for k, v in sc["expect"]["stats"].items():
        assert g["stats"][k] == v, k
    assert [scn.ST[x] for x in sc["expect"]["st"]] == list(g["st"])
    assert list(g["contents"]) == scn.expected_contents(sc)


@pytest.mark.parametrize("seed", range(12))
@pytest.mark.parametrize("mode", ["base", "eager", "lazy"])
def test_small_random(seed, mode):
    rng = np.random.default_rng(seed)
    nb, nf = int(rng.integers(2, 24)), int(rng.integers(1, 6))
    t = tg.gen_small(seed, nblocks=nb, nframes=nf, n_ops=300, max_ranges=4, max_blocks=6)
    assert_parity(t, mode)


@pytest.mark.parametrize("seed", [0, 1, 2])
@pytest.mark.parametrize("mode", ["base", "eager", "lazy"])
def test_c1(seed, mode):
    """C1 tiny (BASELINE.json configs[0]): 64 MiB arena, 16 MiB budget, 64 KiB blocks, 10k ops."""
    assert_parity(tg.gen_c1(seed), mode)


@pytest.mark.parametrize("mode", ["base", "eager", "lazy"])
def test_c1_copy_engine_path(mode):
    """The same C1 trace with every transfer through K4-CE (device plan, copy engines)."""
    t = tg.gen_c1(3).slice_ops(0, 4000)
    assert_parity(t, mode, _gpu(t, mode, copy="ce"))


@pytest.mark.parametrize("mode", ["base", "eager", "lazy"])
def test_c2_ci(mode):
    """C2 streaming at CI size: F = 2048 frames of 2 MiB (4 GiB), buffer 8 GiB, c = 512, P = 2;
    also pins the closed form."""
    F, c, P, B = 2048, 512, 2, 2 << 20
    t = tg.gen_c2(F, c, P, block_bytes=B)
    g, _ = assert_parity(t, mode)
    assert_parity(t, mode, _gpu(t, mode, copy="kernel"))
    s = g["stats"]
    if mode == "base":
        assert (s["h2d_bytes"], s["d2h_bytes"], s["zf_bytes"]) == (2 * (P - 1) * F * B, (2 * P - 1) * F * B, 2 * F * B)
    else:
        assert (s["h2d_bytes"], s["d2h_bytes"], s["zf_bytes"]) == (0, 0, 2 * P * F * B)


@pytest.mark.parametrize("mode", ["base", "eager", "lazy"])
def test_c3_small(mode):
    """C3 (Listing 6) with a VGG-shaped profile scaled down: 2 iterations, 64 KiB blocks."""
    t = tg.gen_c3(block_bytes=64 << 10, budget_bytes=192 << 20, iterations=2, workspace_bytes=4 << 20,
                  layers=tg.scale_layers(tg.VGG16, 1.0 / 512, 1.0 / 64), batch=8)
    assert t.arena_bytes > t.budget_bytes
    for copy in ("default", "ce"):
        assert_parity(t, mode, _gpu(t, mode, copy=copy))


def test_split_large_op():
    """One touch covering 4x the frame budget (ascending sub-ops, A3) and a prefetch of
    the whole arena; ragged tails across many scan tiles."""
    B = 64 << 10
    tb = tg.TraceBuilder(B, 9000 * B, 2100 * B)
    tb.touch([(0, 9000 * B - 100, tg.ACC_WRITE), (5 * B + 7, 3 * B, tg.ACC_READ)])
    tb.discard(100 * B, 4000 * B, lazy_ok=True)
    tb.prefetch(0, 9000 * B, tg.DST_GPU)
    tb.touch([(B * 8000, 900 * B, tg.ACC_WRITE)])
    tb.evict(1500 * B)
    tb.prefetch(0, 3000 * B, tg.DST_HOST)
    t = tb.build()
    for mode in ("base", "eager", "lazy"):
        for copy in ("kernel", "ce"):
            assert_parity(t, mode, _gpu(t, mode, copy=copy))


def test_edge_cases_and_errors():
    from paper_conf_iiswc_zhucvhcr22_b200 import harness, um
    B = 4096
    tb = tg.TraceBuilder(B, 8 * B, 3 * B)
    tb.touch([])                              # empty batch: consumes a seq
    tb.prefetch(0, 0, tg.DST_GPU)             # len 0
    tb.discard(B + 1, B)                      # covers no full block
    tb.evict(0)
    tb.touch([(0, 8 * B, tg.ACC_WRITE)])
    tb.evict(100 * B)                         # more than resident: evict everything
    tb.prefetch(7 * B, B, tg.DST_HOST)
    t = tb.build()
    assert_parity(t, "eager")
    a = harness.make_arena(t, "eager")
    try:
        with pytest.raises(um.UmError) as e:
            um.um_prefetch(a.handle, 7 * B, 2 * B, um.UM_DST_GPU)
        assert e.value.status == um.UM_EINVAL
        with pytest.raises(um.UmError):
            um.um_prefetch(a.handle, 0, B, 5)
        with pytest.raises(um.UmError):
            um.um_touch_batch(a.handle, np.array([(0, B, 1), (8 * B, 1, 1)], dtype=tg.ACC_DTYPE))
        with pytest.raises(um.UmError):
            um.um_alloc(a.handle, 9 * B)
        assert um.um_get_stats(a.handle)["ops"] == 0     # rejected calls enqueue nothing
    finally:
        a.close()


class _CAI:
    def __init__(self, ptr, n, typestr="<u4"):
        self.__cuda_array_interface__ = {"shape": (n,), "typestr": typestr, "data": (ptr, False), "version": 3}


def test_block_table_maps_resident_blocks():
    """D1: map[b] is the frame while G/GL, NONE otherwise (an eager discard unmaps, PAPER
    L176; a lazy discard keeps the mapping, L186); an app kernel can translate through it."""
    import torch
    from paper_conf_iiswc_zhucvhcr22_b200 import harness, um
    B = 64 << 10
    tb = tg.TraceBuilder(B, 16 * B, 8 * B)
    tb.touch([(0, 8 * B, tg.ACC_WRITE)])
    tb.discard(0, 2 * B)
    tb.discard(2 * B, 2 * B, lazy_ok=True)
    t = tb.build()
    a = harness.make_arena(t, "lazy")
    try:
        harness.issue(a, t, "lazy")
        st = um.um_dump(a.handle, a.nblocks, a.nframes)["st"]
        m = torch.as_tensor(_CAI(um.um_block_table(a.handle), a.nblocks, "<i4"), device="cuda").cpu().numpy()
        m = m.astype(np.int64) & 0xFFFFFFFF
        assert [um.ST_NAMES[x] for x in st[:8]] == ["GE", "GE", "GL", "GL", "G", "G", "G", "G"]
        assert (m[:2] == um.UM_NONE).all() and (m[2:8] != um.UM_NONE).all() and (m[8:] == um.UM_NONE).all()
        assert len(set(m[2:8].tolist())) == 6
        # translate block 5 through the table and read its stamp pattern from the frame
        fr = int(m[5])
        blk = a.frames[fr * B:(fr + 1) * B].view(torch.int64).cpu().numpy()
        s = (1 << 32) | 5
        assert blk[0] == s and blk[1] == ~s
    finally:
        a.close()


@pytest.mark.parametrize("mode", ["base", "eager"])
def test_c3_small_tight_host_pool(mode):
    """Host-frame pool sized to the host-resident set (R1/NEXT-4): arena - budget + 2
    blocks.  The fused swap hands the migrating block's host frame to the victim, so the
    pool never needs more than the oracle's max |H| (+ frames freed later in the op)."""
    t = tg.gen_c3(block_bytes=64 << 10, budget_bytes=192 << 20, iterations=2, workspace_bytes=4 << 20,
                  layers=tg.scale_layers(tg.VGG16, 1.0 / 512, 1.0 / 64), batch=8)
    pool = t.arena_bytes - t.budget_bytes + 2 * t.block_bytes
    for copy in ("kernel", "ce"):
        assert_parity(t, mode, _gpu(t, mode, copy=copy, host_pool_bytes=pool))


@pytest.mark.parametrize("ov", [0.8, 2, 4])
@pytest.mark.parametrize("mode", ["base", "eager", "lazy"])
def test_next3_radix_hashjoin(ov, mode):
    MiB = 1 << 20
    B = 64 * 1024
    for t in (tg.gen_radix(block_bytes=B, budget_bytes=int(64 * MiB / ov) // B * B, data_bytes=32 * MiB),
              tg.gen_hashjoin(block_bytes=B, budget_bytes=int(72 * MiB / ov) // B * B, table_bytes=8 * MiB),
              tg.gen_hashjoin(block_bytes=B, budget_bytes=int(72 * MiB / ov) // B * B, table_bytes=8 * MiB,
                              free_at_end=True)):
        assert_parity(t, mode)


@pytest.mark.parametrize("mode", ["base", "eager", "lazy"])
def test_wide_victim_selection(mode):
    """Sub-ops larger than kVictWideMin (8192 blocks) select victims with the multi-CTA
    scan (k_victims_scan/k_victims_apply): large random ranges over 60k blocks with 20k
    frames, interleaved discards (stale ring entries, DISC before USED), big evicts."""
    B = 4096
    base = tg.gen_random(7, block_bytes=B, arena_bytes=60000 * B, budget_bytes=20000 * B, n_ops=50,
                         max_ranges=3, max_blocks=14000, zipf_s=0.3, mix=[50, 20, 5, 10, 10, 0, 5])
    tb = tg.TraceBuilder(B, 60000 * B, 20000 * B)
    for i, (o, fl, off, ln, accs) in enumerate(base.iter_ops()):
        if o == tg.OP_TOUCH:
            tb.touch(accs)
        elif o == tg.OP_PREFETCH:
            tb.prefetch(off, ln, fl)
        elif o == tg.OP_DISCARD:
            tb.discard(off, ln, lazy_ok=bool(fl & 1))
        elif o == tg.OP_HOST_WRITE:
            tb.host_write(off, ln)
        if i % 17 == 16:
            tb.evict(12000 * B)
    t = tb.build()
    for copy in ("kernel", "ce"):
        assert_parity(t, mode, _gpu(t, mode, copy=copy))


@pytest.mark.parametrize("ctas", [1, 3])
def test_wide_victim_scan_tickets(ctas):
    """The same trace with the victim scan grid capped at 1 / 3 CTAs (UM_VS_CTAS, read
    once per process, hence the subprocess): after its first tile every CTA takes tiles
    by ticket and stops past the k-th candidate -- the path full-size tables take (more
    tiles than resident CTAs), here at test size."""
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    code = ("import sys; sys.path[:0] = [%r, %r]; import test_gpu_parity as t\n"
            "for m in ('base', 'eager', 'lazy'): t.test_wide_victim_selection(m)\nprint('ok')") % (root, os.path.join(root, "tests"))
    env = dict(os.environ, UM_VS_CTAS=str(ctas))
    r = subprocess.run([sys.executable, "-c", code], capture_output=True, text=True, timeout=900, cwd=root, env=env)
    assert r.returncode == 0 and r.stdout.strip().endswith("ok"), r.stdout[-2000:] + r.stderr[-4000:]


def _full_size_trace(iterations=2, B=2 << 20):
    import gc
    import torch
    gc.collect()
    torch.cuda.empty_cache()   # the previous full-size test's frames sit in torch's cache
    free, _ = torch.cuda.mem_get_info()
    GiB = 1 << 30
    budget = min(170 * GiB, free - 8 * GiB) // (2 << 20) * (2 << 20)
    assert budget >= 160 * GiB, f"only {free / GiB:.1f} GiB free for the full-size case"
    return tg.gen_c3(block_bytes=B, budget_bytes=budget, oversub=1.5, iterations=iterations)


@pytest.mark.parametrize("mode,copy", [("eager", "default"), ("lazy", "ce"), ("base", "default")])
def test_c3_full_size(mode, copy):
    """Parity at the bench's full size and launch configuration: C3 at 1.5x of a
    170 GiB frame budget (255 GiB arena, 2 MiB blocks), host pool = arena - budget +
    2 GiB, two iterations; every block's state, the queue orders, all counters and every
    block's content tag (frames and host frames read back) against the oracle."""
    t = _full_size_trace()
    pool = t.arena_bytes - t.budget_bytes + (2 << 30)
    g = _gpu(t, mode, copy=copy, host_pool_bytes=pool)
    assert_parity(t, mode, g)
    # north_star: no block moved while discarded (the CUDA path's own transfer log)
    from paper_conf_iiswc_zhucvhcr22_b200 import rmt
    r = rmt.analyze(t, g["xlog"])
    assert r["discarded_state_moves"] == 0
    assert r["h2d_bytes"] == g["stats"]["h2d_bytes"] and r["d2h_bytes"] == g["stats"]["d2h_bytes"]


@pytest.mark.parametrize("pressure", [False, True])
@pytest.mark.parametrize("mode", ["eager", "lazy"])
def test_c4_sweep_cases(pressure, mode):
    """C4 eager-vs-lazy cases (prefix and scattered re-touch) at 64 KiB blocks."""
    for S, p, sc in [(64 << 10, 1.0, False), (32 << 20, 0.5, False), (32 << 20, 0.25, True), (256 << 20, 1.0, False)]:
        t = tg.gen_c4(S, p, block_bytes=64 << 10, pressure=pressure, scattered=sc)
        assert_parity(t, mode)


@pytest.mark.parametrize("seed", [0, 1, 2])
@pytest.mark.parametrize("mode", ["base", "eager", "lazy"])
def test_device_intake(seed, mode):
    """Touch batches of 1-200 unsorted, overlapping ranges with mixed W flags: batches of
    more than 24 records are deduplicated on the device (op bitmap: k_mark, k_runs,
    SURVEY §8(a) A1); distinct blocks often exceed nframes (sub-op splitting)."""
    t = tg.gen_random(seed, block_bytes=64 << 10, arena_bytes=32 << 20, budget_bytes=4 << 20, n_ops=400,
                      max_ranges=200, max_blocks=8, zipf_s=0.8)
    assert_parity(t, mode)


@pytest.mark.parametrize("mode", ["eager", "lazy"])
def test_device_intake_wide(mode):
    """Device-intake batches whose sub-ops exceed 4096 blocks (multi-CTA classify on the
    device-made interval list, wide victim scan) and span several sub-ops."""
    t = tg.gen_random(7, block_bytes=4 << 10, arena_bytes=64 << 20, budget_bytes=24 << 20, n_ops=120,
                      max_ranges=1500, max_blocks=32, zipf_s=0.6)
    assert_parity(t, mode)


# ------------------------------------------------------------------ R7: pipelined app kernels
@pytest.mark.parametrize("seed", range(8))
@pytest.mark.parametrize("mode", ["base", "eager", "lazy"])
def test_overlap_small_random(seed, mode):
    """UM_F_OVERLAP (reading R7): app kernels on their own stream, victim
    selection skipping the last 2 GPU sub-ops' blocks; bit-exact against the oracle's
    window rule, contents included (a hazard would show as a wrong content tag)."""
    rng = np.random.default_rng(100 + seed)
    nb, nf = int(rng.integers(2, 24)), int(rng.integers(1, 6))
    t = tg.gen_small(100 + seed, nblocks=nb, nframes=nf, n_ops=300, max_ranges=4, max_blocks=6)
    assert_parity(t, mode, overlap=True)


@pytest.mark.parametrize("mode", ["base", "eager", "lazy"])
def test_overlap_c1(mode):
    assert_parity(tg.gen_c1(4), mode, overlap=True)


@pytest.mark.parametrize("mode", ["base", "eager", "lazy"])
def test_overlap_c3_small(mode):
    """C3 with pipelined app kernels through every transfer path."""
    t = tg.gen_c3(block_bytes=64 << 10, budget_bytes=192 << 20, iterations=2, workspace_bytes=4 << 20,
                  layers=tg.scale_layers(tg.VGG16, 1.0 / 512, 1.0 / 64), batch=8)
    for copy in ("default", "ce"):
        assert_parity(t, mode, _gpu(t, mode, copy=copy, overlap=True), overlap=True)


@pytest.mark.parametrize("mode", ["eager", "lazy"])
def test_overlap_device_intake(mode):
    """Unsorted batches (device intake rewrites the interval list: waits for app kernels)
    and staged interval lists (stager fences) with pipelined app kernels."""
    t = tg.gen_random(3, block_bytes=64 << 10, arena_bytes=32 << 20, budget_bytes=4 << 20, n_ops=400,
                      max_ranges=200, max_blocks=8, zipf_s=0.8)
    assert_parity(t, mode, overlap=True)
    t = tg.gen_random(7, block_bytes=4 << 10, arena_bytes=64 << 20, budget_bytes=24 << 20, n_ops=120,
                      max_ranges=1500, max_blocks=32, zipf_s=0.6)
    assert_parity(t, mode, overlap=True)


@pytest.mark.parametrize("seed", [0, 1, 2])
@pytest.mark.parametrize("mode", ["base", "eager", "lazy"])
def test_sparse_fault_list(seed, mode):
    """Sparse sorted fault batches (the state microbench's shape at test size): the host
    stages them in the fault-list form (one u32 per block, bit 31 = write); batches span
    many classify tiles, the wide victim scan and several sub-ops."""
    t = tg.gen_sparse(seed)
    assert_parity(t, mode)
    if seed == 0:
        assert_parity(t, mode, _gpu(t, mode, copy="ce"))
        assert_parity(t, mode, overlap=True)


def _sorted_batch_trace(runs, nblocks=4096, nframes=700, B=4 << 10, wfrac=0.5, seed=0):
    """One arena, a few ops whose touch batches are the given lists of (first block,
    run length) records (ascending, disjoint); W on a seeded subset of records."""
    rng = np.random.default_rng(seed)
    tb = tg.TraceBuilder(B, nblocks * B, nframes * B)
    for batch in runs:
        tb.touch([(lo * B, n * B, tg.ACC_WRITE if rng.random() < wfrac else tg.ACC_READ) for lo, n in batch])
        tb.discard(0, (nblocks // 3) * B, lazy_ok=True)
    return tb.build()


@pytest.mark.parametrize("mode", ["eager", "lazy"])
def test_fault_list_boundaries(mode):
    """Edges of the staging choice: 24 records (inline), 25 (staged), runs of exactly 3
    blocks (still the fault-list form) and of 4 (interval form), a list longer than
    nframes (split into sub-ops inside the list), single-block records with alternating
    W flags, adjacent single-block records that merge only where W agrees, and a repeat
    of an earlier batch after a discard of its blocks (revives, revalidations)."""
    gap = lambda n, run, step, base=0: [(base + i * step, run) for i in range(n)]
    batches = [gap(24, 1, 3), gap(25, 1, 3), gap(300, 3, 5), gap(300, 4, 6), gap(1500, 1, 2, 1),
               gap(2000, 1, 2), gap(1000, 1, 1, 2000), gap(25, 1, 3)]
    t = _sorted_batch_trace(batches)
    assert_parity(t, mode)
    assert_parity(t, mode, _gpu(t, mode, copy="kernel"))



@pytest.mark.parametrize("copy", ["default", "ce"])
def test_c3_full_size_64k_blocks(copy):
    """The C3 64 KiB-block variant (~4.18 M blocks, ~2.79 M frames) at full
    size, eager, on the TMA kernel and on per-copy copy engines: two iterations (the trace
    is periodic after the first) bit-exact against the oracle, contents
    included."""
    t = _full_size_trace(iterations=2, B=64 << 10)
    assert t.nblocks > 4_000_000
    pool = t.arena_bytes - t.budget_bytes + (2 << 30)
    g = _gpu(t, "eager", copy=copy, host_pool_bytes=pool, xlog=False)   # ~10 M records: counters only
    assert_parity(t, "eager", g)


@pytest.mark.parametrize("copy", ["default", "ce"])
def test_sparse_d2h_lists(copy):
    """D2H-only lists much shorter than their launch bound (prefetch HOST of mostly
    non-resident ranges, evict of more than is queued): most transfer CTAs get no unit
    and the list must still be reset for the next op (a stale entry would be written
    back again over a reused host frame)."""
    B = 4 << 10
    tb = tg.TraceBuilder(B, 256 * B, 96 * B)
    for r in range(6):
        tb.touch([((r * 7) % 200 * B, 2 * B, tg.ACC_WRITE), ((r * 13 + 100) % 200 * B, B, tg.ACC_WRITE)])
        tb.prefetch(0, 200 * B, tg.DST_HOST)          # 3 resident blocks among 200
        tb.touch([(((r * 5) % 190) * B, 3 * B, tg.ACC_READ | tg.ACC_WRITE)])
        tb.evict(96 * B)                               # more than is queued
        if r == 0:
            tb.prefetch(210 * B, 4 * B, tg.DST_HOST)
            tb.host_write(210 * B, 4 * B)
        tb.touch([(((r * 11) % 150) * B, 4 * B, tg.ACC_READ)])
    t = tb.build()
    for mode in ("base", "eager"):
        assert_parity(t, mode, _gpu(t, mode, copy=copy))


@pytest.mark.parametrize("seed", range(6))
@pytest.mark.parametrize("mode", ["base", "eager", "lazy"])
def test_small_random_with_free(seed, mode):
    """Random traces that also release ranges (um_free, reading R9)."""
    rng = np.random.default_rng(300 + seed)
    nb, nf = int(rng.integers(2, 24)), int(rng.integers(1, 6))
    t = tg.gen_small(300 + seed, nblocks=nb, nframes=nf, n_ops=300, max_ranges=4, max_blocks=6,
                     mix=[45, 12, 5, 10, 10, 3, 2, 13])
    assert_parity(t, mode)


# ------------------------------------------------------------------ R12: proactive eviction
@pytest.mark.parametrize("seed", range(6))
@pytest.mark.parametrize("mode", ["base", "eager", "lazy"])
@pytest.mark.parametrize("overlap", [False, True])
def test_reserve_small_random(seed, mode, overlap):
    """um_config.reserve_blocks (reading R12): after every GPU sub-op the
    engine reclaims frames ahead of demand; bit-exact against the oracle (state, queue
    orders, counters, contents, transfer log), with and without the R7 window."""
    rng = np.random.default_rng(200 + seed)
    nb, nf = int(rng.integers(2, 24)), int(rng.integers(1, 6))
    t = tg.gen_small(200 + seed, nblocks=nb, nframes=nf, n_ops=300, max_ranges=4, max_blocks=6)
    assert_parity(t, mode, overlap=overlap, reserve=int(rng.integers(1, nf + 1)))


@pytest.mark.parametrize("mode", ["base", "eager", "lazy"])
def test_reserve_c1(mode):
    t = tg.gen_c1(5).slice_ops(0, 5000)
    assert_parity(t, mode, reserve=16)
    assert_parity(t, mode, overlap=True, reserve=16)


@pytest.mark.parametrize("mode", ["base", "eager", "lazy"])
def test_reserve_c3_small(mode):
    """C3 with proactive eviction through both transfer paths, sequential and pipelined."""
    t = tg.gen_c3(block_bytes=64 << 10, budget_bytes=192 << 20, iterations=2, workspace_bytes=4 << 20,
                  layers=tg.scale_layers(tg.VGG16, 1.0 / 512, 1.0 / 64), batch=8)
    for copy in ("default", "ce"):
        for ov in (False, True):
            assert_parity(t, mode, _gpu(t, mode, copy=copy, overlap=ov, reserve=64), overlap=ov, reserve=64)


@pytest.mark.parametrize("mode", ["eager", "lazy"])
def test_reserve_wide(mode):
    """A reserve above 8192 frames: the proactive eviction takes the wide victim scan."""
    t = tg.gen_sparse(1, nframes=1 << 14)
    assert_parity(t, mode, reserve=9000)


def test_reserve_rejected():
    """reserve_blocks > nframes, or with two-level granularity: UM_EINVAL."""
    from paper_conf_iiswc_zhucvhcr22_b200 import um
    with pytest.raises(Exception):
        um.Arena(64 << 10, 8 << 20, 4 << 20, reserve_blocks=65, host_pool_bytes=8 << 20)
    with pytest.raises(Exception):
        um.Arena(2 << 20, 64 << 20, 16 << 20, page_bytes=64 << 10, reserve_blocks=1, host_pool_bytes=64 << 20)


# ------------------------------------------------------------------ device-resident records
def _gpu_dev(trace, mode, overlap=False, **kw):
    return _gpu(trace, mode, overlap=overlap, dev_records=True, **kw)


@pytest.mark.parametrize("seed", range(6))
@pytest.mark.parametrize("mode", ["base", "eager", "lazy"])
def test_dev_records_small_random(seed, mode):
    """um_touch_batch_dev: the batch's records read from device memory, range-checked,
    expanded and deduplicated on the GPU (op bitmap -> sorted block list); bit-exact
    against the oracle's touch (state, queue orders, counters, contents, transfer log)."""
    rng = np.random.default_rng(300 + seed)
    nb, nf = int(rng.integers(2, 40)), int(rng.integers(1, 8))
    t = tg.gen_small(300 + seed, nblocks=nb, nframes=nf, n_ops=300, max_ranges=6, max_blocks=6)
    assert_parity(t, mode, _gpu_dev(t, mode))


@pytest.mark.parametrize("mode", ["base", "eager", "lazy"])
def test_dev_records_c1(mode):
    t = tg.gen_c1(6).slice_ops(0, 5000)
    assert_parity(t, mode, _gpu_dev(t, mode))
    assert_parity(t, mode, _gpu_dev(t, mode, overlap=True), overlap=True)
    assert_parity(t, mode, _gpu_dev(t, mode, copy="ce"))
    assert_parity(t, mode, _gpu_dev(t, mode, reserve=8), reserve=8)


@pytest.mark.parametrize("mode", ["eager", "lazy"])
def test_dev_records_unsorted_and_sparse(mode):
    """Unsorted overlapping batches with mixed W flags (1-1500 records), and sparse sorted
    batches spanning many tiles and several sub-ops (the state microbench's shape), over
    arenas whose bitmap ends in a ragged word tile."""
    t = tg.gen_random(3, block_bytes=64 << 10, arena_bytes=(32 << 20) + (37 << 16), budget_bytes=4 << 20,
                      n_ops=400, max_ranges=200, max_blocks=8, zipf_s=0.8)
    assert_parity(t, mode, _gpu_dev(t, mode))
    t = tg.gen_random(7, block_bytes=4 << 10, arena_bytes=64 << 20, budget_bytes=24 << 20, n_ops=120,
                      max_ranges=1500, max_blocks=32, zipf_s=0.6)
    assert_parity(t, mode, _gpu_dev(t, mode))
    t = tg.gen_sparse(2)
    assert_parity(t, mode, _gpu_dev(t, mode))
    assert_parity(t, mode, _gpu_dev(t, mode, overlap=True), overlap=True)


def test_dev_records_range_error_changes_nothing():
    """A device record outside the arena: UM_EINVAL, nothing changed, and the next batch
    (whose bitmap words the rejected one had marked) is serviced exactly."""
    import torch
    from paper_conf_iiswc_zhucvhcr22_b200 import um
    B, nb, nf = 64 << 10, 100, 20
    a = um.Arena(B, nb * B, nf * B, flags=um.UM_F_CHECK, host_pool_bytes=nb * B)
    try:
        h = a.handle
        def dev(recs):
            arr = np.zeros(len(recs), dtype=tg.ACC_DTYPE)
            for i, (o, l, k) in enumerate(recs):
                arr[i] = (o, l, k)
            t = torch.from_numpy(arr.view(np.uint8)).cuda()
            torch.cuda.synchronize()
            return t
        ok = dev([(0, 3 * B, tg.ACC_WRITE), (10 * B, B, tg.ACC_READ)])
        um.um_touch_batch_dev(h, ok.data_ptr(), 2)
        before = um.um_dump(h, nb, nf), um.um_get_stats(h)
        bad = dev([(50 * B, B, tg.ACC_READ), (nb * B - 10, 11, tg.ACC_READ)])
        with pytest.raises(um.UmError) as e:
            um.um_touch_batch_dev(h, bad.data_ptr(), 2)
        assert e.value.status == um.UM_EINVAL
        after = um.um_dump(h, nb, nf), um.um_get_stats(h)
        assert np.array_equal(before[0]["st"], after[0]["st"]) and before[1] == after[1]
        nxt = dev([(60 * B, 2 * B, tg.ACC_READ)])
        um.um_touch_batch_dev(h, nxt.data_ptr(), 1)
        d = um.um_dump(h, nb, nf)
        st = np.asarray(d["st"])
        assert list(np.nonzero(st == 3)[0]) == [0, 1, 2, 10, 60, 61]   # block 50 was never marked in
        with pytest.raises(um.UmError):
            um.um_touch_batch_dev(h, ok.data_ptr() + 8, 1)                # not 16-byte aligned
    finally:
        a.close()


# ------------------------------------------------------------------ the state microbench's op sequence
def _state_micro_parity(t, dev_records, pool=2 << 30):
    g = _gpu(t, "eager", host_pool_bytes=pool, xlog=False, dev_records=dev_records)
    assert_parity(t, "eager", g)
    return g


@pytest.mark.parametrize("dev_records", [False, True])
def test_state_micro_medium(dev_records):
    """bench.py's state microbench sequence at 1/4 size (1 M blocks of 4 KiB, 2/3 of them
    framed, 2^19-record touches): host fault-list and device-record intake, the wide
    victim scan with paced tickets; bit-exact against the oracle."""
    nb = 1 << 20
    t = tg.gen_state_micro(5, block_bytes=4 << 10, arena_bytes=nb * (4 << 10), budget_bytes=(2 * nb // 3) * (4 << 10),
                           n=1 << 19)
    g = _state_micro_parity(t, dev_records, pool=64 << 20)
    assert g["stats"]["evictions"] > 8192


@pytest.mark.parametrize("dev_records", [False, True])
def test_state_micro_full_size(dev_records):
    """The state microbench at its full size and launch configuration (SURVEY §8(d) last
    row: 64 KiB blocks over the bench's 170 GiB budget at 1.5x -> 4.18 M blocks, 2.79 M
    frames; a 2^21-record touch, a discard of 2^21 blocks, a second 2^21-record touch that
    reclaims ~356 k discarded frames), through the host fault list and through
    um_touch_batch_dev: every block's state, both queue orders, all counters and every
    block's content tag against the oracle."""
    import gc
    import torch
    gc.collect()
    torch.cuda.empty_cache()
    free, _ = torch.cuda.mem_get_info()
    GiB = 1 << 30
    budget = min(170 * GiB, free - 8 * GiB) // (2 << 20) * (2 << 20)
    assert budget >= 160 * GiB, f"only {free / GiB:.1f} GiB free for the full-size case"
    arena = int(budget * 1.5) // (2 << 20) * (2 << 20)
    t = tg.gen_state_micro(0, block_bytes=64 << 10, arena_bytes=arena, budget_bytes=budget)
    g = _state_micro_parity(t, dev_records)
    assert g["stats"]["evictions"] > 300_000 and t.nblocks > 4_000_000


def test_dev_records_edge_cases():
    """um_touch_batch_dev edge cases: an empty batch (still one sub-op: the oracle's touch
    of no blocks consumes a seq), zero-length records mixed in, a record covering 100
    blocks across four bitmap words, and UM_EINVAL on a two-level arena."""
    import torch
    from paper_conf_iiswc_zhucvhcr22_b200 import um
    B = 64 << 10
    tb = tg.TraceBuilder(B, 256 * B, 64 * B)
    tb.touch([(5 * B, 0, tg.ACC_WRITE), (7 * B + 3, 10, tg.ACC_WRITE), (30 * B, 100 * B, tg.ACC_READ)])
    tb.touch([])
    tb.touch([(0, 0, tg.ACC_READ)])
    tb.touch([(200 * B, 40 * B, tg.ACC_WRITE), (31 * B, 2 * B, tg.ACC_WRITE)])
    t = tb.build()
    for mode in ("base", "eager"):
        assert_parity(t, mode, _gpu_dev(t, mode))
    a = um.Arena(2 << 20, 64 << 20, 16 << 20, page_bytes=64 << 10, host_pool_bytes=64 << 20)
    try:
        rec = torch.zeros(16, dtype=torch.uint8, device="cuda")
        torch.cuda.synchronize()
        with pytest.raises(um.UmError) as e:
            um.um_touch_batch_dev(a.handle, rec.data_ptr(), 1)
        assert e.value.status == um.UM_EINVAL
    finally:
        a.close()


def test_c3_full_size_reserve():
    """Proactive eviction (R12) at the bench's full size and launch configuration: C3 at
    1.5x of the 170 GiB budget, 2 MiB blocks, reserve 128 frames (the bench's
    proactive-eviction leg), two iterations, bit-exact against the oracle with reserve."""
    t = _full_size_trace()
    pool = t.arena_bytes - t.budget_bytes + (2 << 30)
    g = _gpu(t, "eager", host_pool_bytes=pool, reserve=128)
    assert_parity(t, "eager", g, reserve=128)
