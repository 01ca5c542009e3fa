import os, sys, time
sys.path.insert(0, os.getcwd())
import numpy as np, torch
import tracegen as tg
from paper_conf_iiswc_zhucvhcr22_b200 import um
B = 4096; nb = 4177920; nf = 2785280; n = 1 << 21
a = um.Arena(B, nb * B, nf * B, flags=0, host_pool_bytes=1 << 30)
rng = np.random.default_rng(0)
for rep in range(3):
    blocks = np.sort(rng.choice(nb, size=n, replace=False))
    acc = np.zeros(n, dtype=tg.ACC_DTYPE); acc["off"] = blocks.astype(np.uint64) * B; acc["len"] = B; acc["kind"] = 1
    um.um_get_stats(a.handle)
    t0 = time.perf_counter(); um.um_touch_batch(a.handle, acc); t1 = time.perf_counter()
    print("python-side us", (t1 - t0) * 1e6, flush=True)
    um.um_discard(a.handle, 0, nb * B)
a.close()
