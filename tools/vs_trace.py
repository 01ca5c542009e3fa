"""Timeline of the victim kernels of the pressured touch (tools/state_micro.py's op
sequence: 2^21-block random touch, discard of [0, 2^21), a second random 2^21-block touch
that needs ~356 k victims).  Uses a diagnostic build of libum with -DUM_VS_TRACE
(per-CTA %globaltimer stamps; not the product library):

    nvcc ... -DUM_VS_TRACE -o build/libum_trace.so csrc/um_kernels.cu csrc/um_host.cu
    python tools/vs_trace.py

Prints one JSON line: scan CTAs' start / end spread, tiles per CTA, the finalize span,
apply CTAs' spread (all in microseconds from the first scan CTA's start).
"""
import ctypes
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402
import torch  # noqa: E402

import tracegen as tg  # noqa: E402
from paper_conf_iiswc_zhucvhcr22_b200 import um  # noqa: E402

um.LIB_PATH = os.path.join(ROOT, "build", "libum_trace.so")
B, nb, nf, n = 4096, 4177920, 2785280, 1 << 21
a = um.Arena(B, nb * B, nf * B, flags=um.UM_F_TIMING, host_pool_bytes=1 << 30)
h = a.handle
lib = ctypes.CDLL(um.LIB_PATH)
ps = torch.cuda.ExternalStream(a.stream_ptr)
rng = np.random.default_rng(0)


def records(blocks):
    acc = np.zeros(len(blocks), dtype=tg.ACC_DTYPE)
    acc["off"] = blocks.astype(np.uint64) * B
    acc["len"] = B
    acc["kind"] = tg.ACC_READ
    return acc


def gate():
    with torch.cuda.stream(ps):
        torch.cuda._sleep(100_000_000)


out = []
for rep in range(3):
    if rep:
        a.close()
        a = um.Arena(B, nb * B, nf * B, flags=um.UM_F_TIMING, mem=a.mem)
        h = a.handle
        ps = torch.cuda.ExternalStream(a.stream_ptr)
    acc0 = records(np.sort(rng.choice(nb, size=n, replace=False)))
    acc1 = records(np.sort(rng.choice(nb, size=n, replace=False)))
    um.um_touch_batch(h, acc0)
    um.um_discard(h, 0, n * B)
    torch.cuda.synchronize()
    um.um_timing(h, reset=True)
    gate()
    um.um_touch_batch(h, acc1)
    torch.cuda.synchronize()
    tm = um.um_timing(h, reset=True)
    buf = np.zeros(8192, np.uint64)
    assert lib.um_debug_vs_trace(buf.ctypes.data_as(ctypes.c_void_p), ctypes.c_ulonglong(buf.nbytes)) == 0
    sc = buf[:6000].reshape(-1, 4)
    sc = sc[sc[:, 0] > 0]
    t0 = int(sc[:, 0].min())
    us = lambda x: (np.asarray(x, np.float64) - t0) / 1e3  # noqa: E731
    ap = buf[6000:8000].reshape(-1, 2)
    ap = ap[ap[:, 0] > 0]
    tiles = sc[:, 2].astype(np.int64)
    out.append({
        "rep": rep, "ms_plan": tm["ms_plan"], "scan_ctas": len(sc),
        "scan_start_us": [float(us(sc[:, 0]).min()), float(np.median(us(sc[:, 0]))), float(us(sc[:, 0]).max())],
        "scan_end_us": [float(us(sc[:, 1]).min()), float(np.median(us(sc[:, 1]))), float(us(sc[:, 1]).max())],
        "tiles_per_cta": [int(tiles.min()), float(np.median(tiles)), int(tiles.max()), int(tiles.sum())],
        "first_tile_end_us": [float(us(sc[:, 3]).min()), float(np.median(us(sc[:, 3]))), float(us(sc[:, 3]).max())],
        "finalize_us": [float(us(buf[8000])), float(us(buf[8007])), float(us(buf[8001]))], "examined_tiles": int(buf[8002]), "k": int(buf[8003]),
        "apply_ctas": len(ap),
        "apply_start_us": [float(us(ap[:, 0]).min()), float(us(ap[:, 0]).max())] if len(ap) else None,
        "apply_end_us": [float(us(ap[:, 1]).min()), float(np.median(us(ap[:, 1]))), float(us(ap[:, 1]).max())] if len(ap) else None,
        "victims": um.um_get_stats(h)["evictions"]})
print(json.dumps(out))
a.close()
