"""Hot SASS regions of one profiled kernel instance (stall samples + executed instructions).

    python tools/ncu_sass_hot.py <rep> <kernel-name> [launch-index] [top]
"""
import csv
import io
import subprocess
import sys

rep, name = sys.argv[1], sys.argv[2]
idx = sys.argv[3] if len(sys.argv) > 3 else None
top = int(sys.argv[4]) if len(sys.argv) > 4 else 30
cmd = ["/usr/local/cuda/bin/ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass", "--kernel-name", name]
if idx is not None:
    cmd += ["--launch-skip", idx, "--launch-count", "1"]
out = subprocess.run(cmd, capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
hi = next(i for i, r in enumerate(rows) if r and r[0] == "Address")
h = rows[hi]
R = [r for r in rows[hi + 1:] if len(r) == len(h)]
# a report can list the same function twice; keep the first copy
addrs, first = set(), []
for r in R:
    if r[0] in addrs:
        break
    addrs.add(r[0])
    first.append(r)
R = first


def I(x):
    try:
        return int(x)
    except ValueError:
        return 0


i_s, i_e = h.index("Warp Stall Sampling (All Samples)"), h.index("Instructions Executed")
stalls = [c for c in h if c.startswith("stall_") and "Not Issued" not in c]
print("instructions", sum(I(r[i_e]) for r in R), "samples", sum(I(r[i_s]) for r in R))
agg = {c: sum(I(r[h.index(c)]) for r in R) for c in stalls}
print(sorted(((k[6:], v) for k, v in agg.items() if v), key=lambda x: -x[1]))
for i in sorted(sorted(range(len(R)), key=lambda i: -I(R[i][i_s]))[:top]):
    r = R[i]
    st = {c[6:]: r[h.index(c)] for c in stalls if I(r[h.index(c)]) > 0}
    print(f"{i:5d} {r[1].strip()[:56]:56s} smp {r[i_s]:>4s} exe {r[i_e]:>7s} {st}")
