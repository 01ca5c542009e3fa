"""State-kernel microbench of bench.py's `state_bench` on C3-64K-sized tables without the
170 GiB of frames: 4 KiB blocks, nblocks = 4,177,920, nframes = 2^21 + 2^20 (12 GiB of
frames; 2,785,280 frames as in the bench).  Ops: a touch of 2^21 distinct random blocks (all U, k = 0), a discard of blocks
[0, 2^21), a second random 2^21-block touch under pressure (revives, zero-fills, victims
from DISC).  Prints per-op planning / transfer ms (CUDA-event spans).

    python tools/state_micro.py
    ncu --set full -k regex:'k_classify|k_directive|k_victims' -c 8 python tools/state_micro.py
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
nf = 2785280   # the bench's C3-64K frame count: the pressured touch needs ~356 k victims
n = 1 << 21
a = um.Arena(B, nb * B, nf * B, flags=um.UM_F_TIMING, host_pool_bytes=1 << 30)
h = a.handle
# a device sleep ahead of each op keeps the GPU behind the host: every launch of the op is
# queued before it runs and the spans hold device time only
_ps = torch.cuda.ExternalStream(a.stream_ptr)


def gate():
    with torch.cuda.stream(_ps):
        torch.cuda._sleep(100_000_000)


rng = np.random.default_rng(0)
out = {}


def records(blocks):
    acc = np.zeros(len(blocks), dtype=tg.ACC_DTYPE)
    acc["off"] = blocks.astype(np.uint64) * B
    acc["len"] = B
    acc["kind"] = tg.ACC_READ
    return acc


for rep in range(2):
    acc0 = records(np.sort(rng.choice(nb, size=n, replace=False)))
    acc1 = records(np.sort(rng.choice(nb, size=n, replace=False)))
    if rep:
        a.close()
        a = um.Arena(B, nb * B, nf * B, flags=um.UM_F_TIMING, mem=a.mem)
        h = a.handle
        _ps = torch.cuda.ExternalStream(a.stream_ptr)
    um.um_timing(h, reset=True)
    gate()
    um.um_touch_batch(h, acc0)
    out[f"touch_{rep}"] = um.um_timing(h, reset=True)
    gate()
    um.um_discard(h, 0, n * B)
    out[f"discard_{rep}"] = um.um_timing(h, reset=True)
    gate()
    um.um_touch_batch(h, acc1)
    out[f"touch_pressure_{rep}"] = um.um_timing(h, reset=True)
out["stats"] = um.um_get_stats(h)
print(json.dumps(out))
a.close()
