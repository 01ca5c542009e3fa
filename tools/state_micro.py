"""State-kernel microbench on C3-64K-sized tables without the 170 GiB of frames:
4 KiB blocks, nblocks = 4,177,920, nframes = 2^21 + 2^20 (frames 12 GiB), one touch of
2^21 distinct random blocks (all U -> zero-fill), one 2^21-block discard, a prefetch of
the discarded range (revive) and a second random touch under pressure.

    python tools/state_micro.py            # prints per-op planning / transfer ms
    ncu --set full -k regex:'k_classify|k_directive' -c 4 python tools/state_micro.py
"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import tracegen as tg  # noqa: E402
from paper_conf_iiswc_zhucvhcr22_b200 import build, um  # noqa: E402

build.build()
B = 4096
nb = 4177920
nf = (1 << 21) + (1 << 20)
n = 1 << 21
a = um.Arena(B, nb * B, nf * B, flags=um.UM_F_TIMING | um.UM_F_COPY_KERNEL, host_pool_bytes=1 << 30)
h = a.handle
# Gate: a ~50 ms device sleep on the paging stream before each op, so every launch of the
# op is queued before the GPU reaches it and the timed spans hold device time only (no
# host enqueue gaps between the kernels).
_ps = torch.cuda.ExternalStream(a.stream_ptr)


def gate():
    with torch.cuda.stream(_ps):
        torch.cuda._sleep(100_000_000)
rng = np.random.default_rng(0)
out = {}


def touch_random(tag):
    blocks = np.sort(rng.choice(nb, size=n, replace=False))
    acc = np.zeros(n, dtype=tg.ACC_DTYPE)
    acc["off"] = blocks.astype(np.uint64) * B
    acc["len"] = B
    acc["kind"] = tg.ACC_READ
    um.um_timing(h, reset=True)
    gate()
    um.um_touch_batch(h, acc)
    out[tag] = um.um_timing(h, reset=True)


for rep in range(2):
    touch_random(f"touch_random_{rep}")
    gate()
    um.um_discard(h, 0, n * B)
    out[f"discard_{rep}"] = um.um_timing(h, reset=True)
    gate()
    um.um_prefetch(h, 0, n * B, um.UM_DST_GPU)
    out[f"prefetch_revive_{rep}"] = um.um_timing(h, reset=True)
out["stats"] = um.um_get_stats(h)
print(json.dumps(out))
a.close()
