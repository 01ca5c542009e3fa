"""CPU checks of the C-ABI boundary: libum.so builds for sm_100a, loads without a GPU,
and exports every function include/um.h declares; host-side interval logic."""
import os
import re
import subprocess

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HDR = os.path.join(ROOT, "include", "um.h")


def _declared():
    src = open(HDR).read()
    return sorted(set(re.findall(r"\b(um_[a-z_]+)\s*\(", src)))


def test_build_and_exports():
    from paper_conf_iiswc_zhucvhcr22_b200 import build, um
    lib = build.build()
    names = _declared()
    assert "um_discard_lazy" in names and "um_touch_batch" in names
    L = um.lib()
    for n in names:
        assert hasattr(L, n), n
    assert set(um.EXPORTS) == set(names)
    out = subprocess.run(["nm", "-D", "--defined-only", lib], capture_output=True, text=True).stdout
    exported = set(re.findall(r"\bT (um_[a-z_]+)", out))
    assert exported == set(names), exported ^ set(names)


def test_sass_is_sm100a_and_uses_tma():
    from paper_conf_iiswc_zhucvhcr22_b200 import build
    lib = build.build()
    sass = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "-sass", lib], capture_output=True, text=True).stdout
    assert "sm_100a" in sass
    assert "UBLKCP" in sass          # cp.async.bulk (TMA bulk copy) in the transfer engine
    assert "SYNCS" in sass           # mbarrier


def test_strerror_without_gpu():
    from paper_conf_iiswc_zhucvhcr22_b200 import um
    assert um.um_strerror(um.UM_EINVAL) == "invalid argument"
    assert um.um_strerror(um.UM_OK) == "ok"


def test_workspace_size_and_config_validation_without_gpu():
    import ctypes as C
    from paper_conf_iiswc_zhucvhcr22_b200 import um
    hc = (C.c_void_p * 1)(1)
    cfg = um.um_config(device=0, block_bytes=65536, arena_bytes=64 << 20, budget_bytes=16 << 20, frames=None,
                       workspace=None, workspace_bytes=0, host_chunks=C.cast(hc, C.POINTER(C.c_void_p)),
                       n_host_chunks=1, host_chunk_bytes=64 << 20, flags=0)
    ws = um.um_workspace_size(cfg)
    assert ws > 1024 * 1 + 21 * 1024
    bad = um.um_config.from_buffer_copy(cfg)
    bad.arena_bytes = (64 << 20) + 1
    with pytest.raises(um.UmError):
        um.um_workspace_size(bad)
    bad = um.um_config.from_buffer_copy(cfg)
    bad.block_bytes = 3000
    with pytest.raises(um.UmError):
        um.um_workspace_size(bad)
    # arena_create rejects missing memory before touching the GPU
    out = C.c_void_p()
    assert um.lib().um_arena_create(C.byref(cfg), C.byref(out)) == um.UM_EINVAL


def test_two_level_config_validation_without_gpu():
    """page_bytes: 0 or block_bytes = single level; otherwise a power of
    two >= 16 KiB with <= 32 pages per block, not with UM_F_COPY_CE / UM_F_OVERLAP."""
    import ctypes as C
    from paper_conf_iiswc_zhucvhcr22_b200 import um
    hc = (C.c_void_p * 1)(1)
    base = um.um_config(device=0, block_bytes=2 << 20, arena_bytes=64 << 20, budget_bytes=16 << 20, frames=None,
                        workspace=None, workspace_bytes=0, host_chunks=C.cast(hc, C.POINTER(C.c_void_p)),
                        n_host_chunks=1, host_chunk_bytes=64 << 20, flags=0, page_bytes=0)
    ws1 = um.um_workspace_size(base)
    ok = um.um_config.from_buffer_copy(base)
    ok.page_bytes = 64 << 10
    assert um.um_workspace_size(ok) > ws1          # page masks and per-page tags
    same = um.um_config.from_buffer_copy(base)
    same.page_bytes = 2 << 20
    assert um.um_workspace_size(same) == ws1
    for pb, fl in [(32 << 10, 0), (48 << 10, 0), (8 << 10, 0), (64 << 10, um.UM_F_COPY_CE), (64 << 10, 64)]:
        bad = um.um_config.from_buffer_copy(base)
        bad.page_bytes, bad.flags = pb, fl
        with pytest.raises(um.UmError):
            um.um_workspace_size(bad)


def test_reserve_config_validation_without_gpu():
    """reserve_blocks (R12 proactive eviction): accepted up to nframes at single level;
    above nframes, or with two-level page_bytes, UM_EINVAL."""
    import ctypes as C
    from paper_conf_iiswc_zhucvhcr22_b200 import um
    hc = (C.c_void_p * 1)(1)
    base = um.um_config(device=0, block_bytes=2 << 20, arena_bytes=64 << 20, budget_bytes=16 << 20, frames=None,
                        workspace=None, workspace_bytes=0, host_chunks=C.cast(hc, C.POINTER(C.c_void_p)),
                        n_host_chunks=1, host_chunk_bytes=64 << 20, flags=0, page_bytes=0)
    ws = um.um_workspace_size(base)
    for r in (1, 8):
        ok = um.um_config.from_buffer_copy(base)
        ok.reserve_blocks = r
        assert um.um_workspace_size(ok) == ws
    for r, pb in [(9, 0), (1, 64 << 10)]:
        bad = um.um_config.from_buffer_copy(base)
        bad.reserve_blocks, bad.page_bytes = r, pb
        with pytest.raises(um.UmError):
            um.um_workspace_size(bad)
