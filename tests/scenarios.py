"""Parser for tests/golden/scenarios.yaml -> tracegen.Trace + expected values.
Shared by the oracle pins (CPU) and the CUDA parity tests (GPU).  Test code only."""
import os

import yaml

import tracegen as tg

GOLDEN = os.path.join(os.path.dirname(__file__), "golden", "scenarios.yaml")
ST = {"U": 0, "H": 1, "HD": 2, "G": 3, "GE": 4, "GL": 5}


def load():
    with open(GOLDEN) as f:
        return yaml.safe_load(f)


def _blocks(spec):
    if "-" in spec:
        lo, hi = spec.split("-")
        return int(lo), int(hi)
    return int(spec), int(spec)


def build(sc) -> tuple:
    """Returns (trace, mode, ops_modes) where the DISCARD records of the trace carry
    lazy_ok=1 exactly for 'discard_lazy' lines; run it in mode sc['mode'] (lazy mode
    turns lazy_ok discards into UvmDiscardLazy)."""
    B, nb, nf = sc["B"], sc["nblocks"], sc["nframes"]
    tb = tg.TraceBuilder(B, nb * B, nf * B)
    for line in sc["ops"]:
        w = line.split()
        op = w[0]
        if op == "touch":
            accs = []
            for part in w[1].split(","):
                r, k = part.split(":")
                lo, hi = _blocks(r)
                kind = {"R": tg.ACC_READ, "W": tg.ACC_WRITE, "RW": tg.ACC_READ | tg.ACC_WRITE}[k]
                accs.append((lo * B, (hi - lo + 1) * B, kind))
            tb.touch(accs)
        elif op == "prefetch":
            lo, hi = _blocks(w[1])
            tb.prefetch(lo * B, (hi - lo + 1) * B, tg.DST_GPU if w[2] == "GPU" else tg.DST_HOST)
        elif op in ("discard", "discard_lazy"):
            lo, hi = _blocks(w[1])
            tb.discard(lo * B, (hi - lo + 1) * B, lazy_ok=(op == "discard_lazy"))
        elif op == "discard_bytes":
            tb.discard(int(w[1]), int(w[2]))
        elif op == "evict":
            tb.evict(int(w[1]) * B)
        elif op == "free":
            lo, hi = _blocks(w[1])
            tb.free(lo * B, (hi - lo + 1) * B)
        elif op == "evict_bytes":
            tb.evict(int(w[1]))
        elif op == "touch_bytes":
            kind = {"R": tg.ACC_READ, "W": tg.ACC_WRITE, "RW": tg.ACC_READ | tg.ACC_WRITE}[w[3]]
            tb.touch([(int(w[1]), int(w[2]), kind)])
        elif op == "prefetch_bytes":
            tb.prefetch(int(w[1]), int(w[2]), tg.DST_GPU if w[3] == "GPU" else tg.DST_HOST)
        elif op == "host_write":
            lo, hi = _blocks(w[1])
            tb.host_write(lo * B, (hi - lo + 1) * B)
        else:
            raise ValueError(line)
    return tb.build(), sc["mode"]


def expected_contents(sc):
    """'s<k>' -> stamp(seq=k, block) = (k << 32) | block; '0' -> 0."""
    out = []
    for b, c in enumerate(sc["expect"]["contents"]):
        out.append(0 if c in (0, "0") else (int(str(c)[1:]) << 32) | b)
    return out
