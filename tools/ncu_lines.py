"""Per-source-line warp-stall samples of one kernel in an ncu report (run here, no GPU).

    python tools/ncu_lines.py <report.ncu-rep> <kernel regex> [launch_skip] [top]
"""
import csv
import io
import subprocess
import sys

rep, kern = sys.argv[1], sys.argv[2]
skip = sys.argv[3] if len(sys.argv) > 3 else "0"
top = int(sys.argv[4]) if len(sys.argv) > 4 else 20
out = subprocess.run(["/usr/local/cuda/bin/ncu", "-i", rep, "--page", "source", "--csv", "--kernel-name", f"regex:{kern}",
                      "--launch-skip", skip, "--launch-count", "1", "--print-source", "sass,cuda"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
agg, cur = {}, None
for r in rows[3:]:
    if len(r) < 6:
        continue
    if r[0] != "":
        cur = (r[0], r[1].strip()[:100])
        try:
            agg[cur] = agg.get(cur, 0) + int(r[4])
        except ValueError:
            pass
tot = sum(agg.values())
print(f"total samples {tot}")
for k, v in sorted(agg.items(), key=lambda x: -x[1])[:top]:
    print(f"{v:6d} {100.0 * v / max(tot, 1):5.1f}%  L{k[0]}: {k[1]}")
