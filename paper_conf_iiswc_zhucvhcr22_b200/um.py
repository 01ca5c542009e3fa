"""Thin ctypes binding of libum (include/um.h): same names, argument marshalling only.

Every step of the paging path runs in libum's sm_100a kernels; this module only
converts Python values to C arguments.  It raises loudly if libum.so is missing —
there is no CPU fallback.  PyTorch is used only to allocate device memory, pinned
host memory and streams (the `Arena` helper at the bottom).
"""
from __future__ import annotations

import ctypes as C
import os

import numpy as np

_PKG = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_PKG, "libum.so")

UM_OK, UM_EINVAL, UM_ENOMEM, UM_ECUDA, UM_EBUSY = 0, -1, -2, -3, -4
UM_DST_GPU, UM_DST_HOST = 0, 1
UM_ACC_READ, UM_ACC_WRITE = 1, 2
UM_ST_U, UM_ST_H, UM_ST_HD, UM_ST_G, UM_ST_GE, UM_ST_GL = range(6)
ST_NAMES = ("U", "H", "HD", "G", "GE", "GL")
UM_F_DISCARD_OFF, UM_F_COPY_CE, UM_F_CHECK, UM_F_APP_STAMP, UM_F_TIMING, UM_F_COPY_KERNEL = 1, 2, 4, 8, 16, 32
UM_F_OVERLAP = 64
UM_NONE = 0xFFFFFFFF


class um_access(C.Structure):
    _fields_ = [("off", C.c_uint64), ("len", C.c_uint32), ("kind", C.c_uint32)]


class um_config(C.Structure):
    _fields_ = [("device", C.c_int), ("block_bytes", C.c_uint32), ("arena_bytes", C.c_uint64),
                ("budget_bytes", C.c_uint64), ("frames", C.c_void_p), ("workspace", C.c_void_p),
                ("workspace_bytes", C.c_uint64), ("host_chunks", C.POINTER(C.c_void_p)),
                ("n_host_chunks", C.c_uint32), ("host_chunk_bytes", C.c_uint64), ("flags", C.c_uint32),
                ("page_bytes", C.c_uint32), ("reserve_blocks", C.c_uint32)]


STAT_FIELDS = ("h2d_bytes", "d2h_bytes", "zf_bytes", "h2d_avoided_bytes", "d2h_avoided_bytes", "faults",
               "hits", "remaps", "unmaps", "revalidations", "refreshes", "evictions", "ops", "subops")


class um_stats(C.Structure):
    _fields_ = [(n, C.c_int64) for n in STAT_FIELDS] + [("pad", C.c_int64 * 2)]

    def as_dict(self):
        return {n: int(getattr(self, n)) for n in STAT_FIELDS}


class UmError(RuntimeError):
    def __init__(self, fn, status):
        super().__init__(f"{fn} failed: {status} ({um_strerror(status)})")
        self.status = status


_lib = None


def lib():
    """Load libum.so (raises if it was not built — no fallback)."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise ImportError(f"{LIB_PATH} missing: run `python -m paper_conf_iiswc_zhucvhcr22_b200.build`")
        L = C.CDLL(LIB_PATH)
        P, U64, U32, I = C.c_void_p, C.c_uint64, C.c_uint32, C.c_int
        sig = {
            "um_workspace_size": [C.POINTER(um_config), C.POINTER(U64)],
            "um_arena_create": [C.POINTER(um_config), C.POINTER(P)],
            "um_arena_destroy": [P],
            "um_alloc": [P, U64, C.POINTER(U64)],
            "um_prefetch": [P, U64, U64, I, P],
            "um_discard": [P, U64, U64, P],
            "um_discard_lazy": [P, U64, U64, P],
            "um_touch_batch": [P, P, U32, P],
            "um_touch_batch_dev": [P, P, U32, P],
            "um_evict": [P, U64, P],
            "um_free": [P, U64, U64, P],
            "um_host_write": [P, U64, U64, P],
            "um_block_table": [P, C.POINTER(P)],
            "um_stream": [P, C.POINTER(P)],
            "um_join": [P, P],
            "um_get_stats": [P, C.POINTER(um_stats)],
            "um_dump": [P, P, P, C.POINTER(U32), P, C.POINTER(U32)],
            "um_content_tags": [P, P],
            "um_timing": [P, C.POINTER(C.c_double), C.POINTER(C.c_double), C.POINTER(U64), C.POINTER(U64), I],
            "um_xlog_attach": [P, P, U64],
            "um_xlog_count": [P, C.POINTER(U64)],
            "um_page_masks": [P, P, P],
        }
        for name, args in sig.items():
            f = getattr(L, name)
            f.argtypes = args
            f.restype = C.c_int
        L.um_strerror.argtypes = [C.c_int]
        L.um_strerror.restype = C.c_char_p
        _lib = L
    return _lib


EXPORTS = ("um_workspace_size", "um_arena_create", "um_arena_destroy", "um_alloc", "um_prefetch", "um_discard",
           "um_discard_lazy", "um_touch_batch", "um_touch_batch_dev", "um_evict", "um_free", "um_host_write", "um_block_table", "um_stream",
           "um_join", "um_get_stats", "um_dump", "um_content_tags", "um_timing", "um_xlog_attach",
           "um_xlog_count", "um_page_masks", "um_strerror")


def _ck(fn, st):
    if st != UM_OK:
        raise UmError(fn, st)


def um_strerror(status: int) -> str:
    return lib().um_strerror(status).decode()


def um_workspace_size(cfg: um_config) -> int:
    out = C.c_uint64()
    _ck("um_workspace_size", lib().um_workspace_size(C.byref(cfg), C.byref(out)))
    return out.value


def um_arena_create(cfg: um_config) -> int:
    out = C.c_void_p()
    _ck("um_arena_create", lib().um_arena_create(C.byref(cfg), C.byref(out)))
    return out.value


def um_arena_destroy(a) -> None:
    _ck("um_arena_destroy", lib().um_arena_destroy(a))


def um_alloc(a, nbytes: int) -> int:
    off = C.c_uint64()
    _ck("um_alloc", lib().um_alloc(a, nbytes, C.byref(off)))
    return off.value


def um_prefetch(a, off: int, ln: int, dst: int, stream=None) -> None:
    _ck("um_prefetch", lib().um_prefetch(a, off, ln, dst, stream))


def um_discard(a, off: int, ln: int, stream=None) -> None:
    _ck("um_discard", lib().um_discard(a, off, ln, stream))


def um_discard_lazy(a, off: int, ln: int, stream=None) -> None:
    _ck("um_discard_lazy", lib().um_discard_lazy(a, off, ln, stream))


def um_touch_batch(a, acc: np.ndarray, stream=None) -> None:
    """acc: numpy array with the 16-byte um_access layout (tracegen.ACC_DTYPE)."""
    acc = np.ascontiguousarray(acc)
    assert acc.dtype.itemsize == 16
    _ck("um_touch_batch", lib().um_touch_batch(a, acc.ctypes.data if len(acc) else None, len(acc), stream))


def um_touch_batch_dev(a, acc_ptr: int, n: int, stream=None) -> None:
    """acc_ptr: device address of n 16-byte um_access records (16-byte aligned)."""
    _ck("um_touch_batch_dev", lib().um_touch_batch_dev(a, acc_ptr or None, n, stream))


def um_evict(a, nbytes: int, stream=None) -> None:
    _ck("um_evict", lib().um_evict(a, nbytes, stream))


def um_free(a, off: int, ln: int, stream=None) -> None:
    _ck("um_free", lib().um_free(a, off, ln, stream))


def um_host_write(a, off: int, ln: int, stream=None) -> None:
    _ck("um_host_write", lib().um_host_write(a, off, ln, stream))


def um_block_table(a) -> int:
    p = C.c_void_p()
    _ck("um_block_table", lib().um_block_table(a, C.byref(p)))
    return p.value


def um_join(a, stream=None) -> None:
    """Make `stream` (default: the arena's paging stream) wait for all enqueued work,
    including UM_F_OVERLAP application kernels."""
    _ck("um_join", lib().um_join(a, stream if stream is not None else um_stream(a)))


def um_stream(a) -> int:
    p = C.c_void_p()
    _ck("um_stream", lib().um_stream(a, C.byref(p)))
    return p.value


def um_get_stats(a) -> dict:
    s = um_stats()
    _ck("um_get_stats", lib().um_get_stats(a, C.byref(s)))
    return s.as_dict()


def um_dump(a, nblocks: int, nframes: int) -> dict:
    st = np.zeros(nblocks, np.uint8)
    used = np.zeros(max(1, nframes), np.uint32)
    disc = np.zeros(max(1, nframes), np.uint32)
    nu, nd = C.c_uint32(), C.c_uint32()
    _ck("um_dump", lib().um_dump(a, st.ctypes.data, used.ctypes.data, C.byref(nu), disc.ctypes.data, C.byref(nd)))
    return {"st": st, "used_order": used[:nu.value].tolist(), "disc_order": disc[:nd.value].tolist()}


def um_page_masks(a, nblocks: int) -> tuple:
    dead, lazy = np.zeros(nblocks, np.uint32), np.zeros(nblocks, np.uint32)
    _ck("um_page_masks", lib().um_page_masks(a, dead.ctypes.data, lazy.ctypes.data))
    return dead, lazy


def um_content_tags(a, nblocks: int) -> np.ndarray:
    t = np.zeros(nblocks, np.uint64)
    _ck("um_content_tags", lib().um_content_tags(a, t.ctypes.data))
    return t


def um_timing(a, reset: bool = False) -> dict:
    p, x = C.c_double(), C.c_double()
    nx, nl = C.c_uint64(), C.c_uint64()
    _ck("um_timing", lib().um_timing(a, C.byref(p), C.byref(x), C.byref(nx), C.byref(nl), int(reset)))
    return {"ms_plan": p.value, "ms_xfer": x.value, "xfer_launches": nx.value, "launches": nl.value}


XL_KIND = ("H2D", "D2H", "ZF")


def um_xlog_attach(a, dev_ptr, cap_entries: int) -> None:
    _ck("um_xlog_attach", lib().um_xlog_attach(a, dev_ptr, cap_entries))


def um_xlog_count(a) -> int:
    n = C.c_uint64()
    _ck("um_xlog_count", lib().um_xlog_count(a, C.byref(n)))
    return n.value


# -------------------------------------------------------------------------------------
# Arena: allocates the caller-owned memory with torch (frames + workspace in HBM,
# host-frame pool in pinned host memory) and creates the libum arena.
# -------------------------------------------------------------------------------------
class Memory:
    """Caller-owned memory for an arena, allocated once with torch and reusable by
    several arenas in sequence: frames (HBM), workspace (HBM), host-frame pool
    (pinned host memory in chunks of <= 1 GiB, allocated from `threads` threads)."""

    def __init__(self, block_bytes: int, arena_bytes: int, budget_bytes: int, *, host_pool_bytes=None,
                 host_chunk_bytes=None, device: int | None = None, threads: int = 1, page_bytes: int = 0):
        import torch
        if device is None:   # the caller's current device (one process per GPU under torchrun)
            device = torch.cuda.current_device()
        self.B = block_bytes
        self.page_bytes = page_bytes
        self.nframes = budget_bytes // block_bytes
        if host_pool_bytes is None:
            host_pool_bytes = arena_bytes          # every block can be host-resident
        host_pool_bytes += block_bytes             # + the zero page
        if host_chunk_bytes is None:
            host_chunk_bytes = min(1 << 30, max(block_bytes, 1 << (host_pool_bytes - 1).bit_length()))
        self.host_chunk_bytes = host_chunk_bytes
        nch = -(-host_pool_bytes // host_chunk_bytes)
        self.device = device
        dev = torch.device("cuda", device)
        self.frames = torch.empty(self.nframes * block_bytes, dtype=torch.uint8, device=dev)
        mk = lambda _: torch.empty(host_chunk_bytes, dtype=torch.uint8, pin_memory=True)
        if threads > 1 and nch > 1:
            from concurrent.futures import ThreadPoolExecutor
            with ThreadPoolExecutor(threads) as ex:
                self.host_chunks = list(ex.map(mk, range(nch)))
        else:
            self.host_chunks = [mk(i) for i in range(nch)]
        self._hc = (C.c_void_p * nch)(*[t.data_ptr() for t in self.host_chunks])
        probe = um_config(device=device, block_bytes=block_bytes, arena_bytes=arena_bytes,
                          budget_bytes=budget_bytes, frames=self.frames.data_ptr(), workspace=None,
                          workspace_bytes=0, host_chunks=C.cast(self._hc, C.POINTER(C.c_void_p)),
                          n_host_chunks=nch, host_chunk_bytes=host_chunk_bytes, flags=0, page_bytes=page_bytes)
        ws = um_workspace_size(probe)
        self.workspace = torch.empty(ws, dtype=torch.uint8, device=dev)
        self.nch = nch
        # the arena's streams do not wait for torch's stream: hand the memory over only
        # after any pending torch work on it (a previous owner's) is done
        torch.cuda.synchronize(dev)

    def config(self, arena_bytes: int, budget_bytes: int, flags: int) -> um_config:
        return um_config(device=self.device, block_bytes=self.B, arena_bytes=arena_bytes,
                         budget_bytes=budget_bytes, frames=self.frames.data_ptr(),
                         workspace=self.workspace.data_ptr(), workspace_bytes=self.workspace.numel(),
                         host_chunks=C.cast(self._hc, C.POINTER(C.c_void_p)), n_host_chunks=self.nch,
                         host_chunk_bytes=self.host_chunk_bytes, flags=flags, page_bytes=self.page_bytes)


class Arena:
    """A libum arena over `Memory` (allocated here unless `mem` is given)."""

    def __init__(self, block_bytes: int, arena_bytes: int, budget_bytes: int, *, flags: int = 0,
                 host_pool_bytes: int | None = None, host_chunk_bytes: int | None = None, device: int | None = None,
                 mem: Memory | None = None, page_bytes: int = 0, reserve_blocks: int = 0):
        self.B = block_bytes
        self.nblocks = arena_bytes // block_bytes
        self.nframes = budget_bytes // block_bytes
        self.mem = mem if mem is not None else Memory(block_bytes, arena_bytes, budget_bytes,
                                                      host_pool_bytes=host_pool_bytes,
                                                      host_chunk_bytes=host_chunk_bytes, device=device,
                                                      page_bytes=page_bytes)
        self.frames = self.mem.frames
        self.cfg = self.mem.config(arena_bytes, budget_bytes, flags)
        if page_bytes:
            self.cfg.page_bytes = page_bytes
        self.cfg.reserve_blocks = reserve_blocks   # R12 proactive eviction (0: on demand only)
        self.ppc = block_bytes // self.cfg.page_bytes if self.cfg.page_bytes else 1
        self.handle = um_arena_create(self.cfg)
        self.stream_ptr = um_stream(self.handle)

    def close(self):
        if self.handle:
            um_arena_destroy(self.handle)
            self.handle = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass
