"""B200-native discard-aware unified-memory paging layer (UVM Discard, Zhu et al. IISWC'22).

The product is libum.so (C ABI in include/um.h, sm_100a kernels in csrc/); `um` is
its thin ctypes binding and `harness` replays tracegen traces through it.
"""
from . import um  # noqa: F401
