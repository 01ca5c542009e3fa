"""How fast can one kernel stream a few tens of MB on this GPU?  Times torch's own
kernels (sum = read-only, clone = copy, zero_ = write) over 8-256 MB buffers with cold
L2 (a 512 MB scrub between reps), CUDA events, median of 20.  Context for the state
kernels, which move 30-60 MB per launch."""
import json
import statistics

import torch

dev = torch.device("cuda", 0)
scrub = torch.empty(512 << 20, dtype=torch.uint8, device=dev)
out = []
for mb in (8, 16, 32, 64, 128, 256):
    x = torch.ones((mb << 20) // 8, dtype=torch.int64, device=dev)
    y = torch.empty_like(x)
    row = {"mb": mb}
    for name, fn, factor in (("read_sum", lambda: x.sum(), 1), ("copy", lambda: y.copy_(x), 2), ("write_zero", lambda: y.zero_(), 1)):
        ts = []
        for _ in range(21):
            scrub.add_(1)
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            fn()
            e1.record()
            e1.synchronize()
            ts.append(e0.elapsed_time(e1))
        t = statistics.median(ts[1:])
        row[name] = {"us": t * 1e3, "gbs": factor * (mb << 20) / (t / 1e3) / 1e9}
    out.append(row)
print(json.dumps(out))
