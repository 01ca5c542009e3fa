"""Summarise ncu outputs into markdown for profiles/ (run here, no GPU needed).

    python tools/ncu_summary.py launches <launches.csv>
    python tools/ncu_summary.py report <file.ncu-rep> [...]
"""
import collections
import csv
import io
import subprocess
import sys

NCU = "/usr/local/cuda/bin/ncu"


def launches(path):
    rows = list(csv.reader(open(path)))
    hi = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
    h = rows[hi]
    ki, vi, ui = h.index("Kernel Name"), h.index("Metric Value"), h.index("Metric Unit")
    mi = h.index("Metric Name") if "Metric Name" in h else None
    tot, cnt = collections.defaultdict(float), collections.Counter()
    scale = {"ns": 1e-6, "nsecond": 1e-6, "us": 1e-3, "usecond": 1e-3, "ms": 1.0, "msecond": 1.0}
    for r in rows[hi + 1:]:
        if len(r) <= vi or not r[vi]:
            continue
        if mi is not None and r[mi] != "gpu__time_duration.sum":
            continue
        name = r[ki].split("(")[0]
        tot[name] += float(r[vi].replace(",", "")) * scale.get(r[ui], 1.0)
        cnt[name] += 1
    T = sum(tot.values())
    out = ["| kernel | launches | total ms | share | avg ms |", "|---|---:|---:|---:|---:|"]
    for k, v in sorted(tot.items(), key=lambda x: -x[1]):
        out.append(f"| {k} | {cnt[k]} | {v:.2f} | {v / T:.4f} | {v / cnt[k]:.4f} |")
    return "\n".join(out)


KEYS = [("gpu__time_duration.sum", "dur"), ("dram__bytes_read.sum", "dram rd"), ("dram__bytes_write.sum", "dram wr"),
        ("gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "dram %"),
        ("pcie__read_bytes.sum.per_second", "pcie rd/s"), ("pcie__write_bytes.sum.per_second", "pcie wr/s"),
        ("sm__throughput.avg.pct_of_peak_sustained_elapsed", "sm %"),
        ("launch__grid_size", "grid"), ("launch__block_size", "block"),
        ("launch__registers_per_thread", "regs"), ("sm__warps_active.avg.pct_of_peak_sustained_active", "warps act %")]


def report(path):
    raw = subprocess.run([NCU, "-i", path, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(raw)))
    h, u = rows[0], rows[1]
    ki = h.index("Kernel Name")
    cols = [(h.index(k), lab) for k, lab in KEYS if k in h]
    out = ["| kernel | " + " | ".join(lab for _, lab in cols) + " |", "|---|" + "---:|" * len(cols)]
    for r in rows[2:]:
        out.append(f"| {r[ki].split('(')[0]} | " + " | ".join(f"{r[i]} {u[i]}".strip() for i, _ in cols) + " |")
    return "\n".join(out)


if __name__ == "__main__":
    if sys.argv[1] == "launches":
        print(launches(sys.argv[2]))
    else:
        for p in sys.argv[2:]:
            print(f"\n### {p}\n")
            print(report(p))
