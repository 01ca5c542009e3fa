"""Summarise the k_service traffic capture of tools/ncu_round.sh (step 2) into JSON for
profiles/ (run here, no GPU):

    python tools/service_traffic.py gpurun_out/ncu/service_traffic.csv gpurun_out/ncu/traffic.log > profiles/r02_service_traffic.json

The capture holds every k_service launch of the bench's timed C3 iteration (eager); the
bench line printed in traffic.log gives that iteration's counters, i.e. the algorithmic
bytes: link = H2D + D2H (what crosses PCIe), HBM = H2D + D2H + zero-fill (frame writes
and reads).  ncu's pcie__*_bytes count at 512 B granularity, dram__bytes at 32 B sectors.
"""
import collections
import csv
import json
import sys


def main(csv_path, log_path):
    rows = list(csv.reader(open(csv_path)))
    hi = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
    h = rows[hi]
    ix = {k: h.index(k) for k in ("ID", "Metric Name", "Metric Value", "Metric Unit")}
    per = collections.defaultdict(dict)
    for r in rows[hi + 1:]:
        if len(r) < len(h):
            continue
        per[int(r[ix["ID"]])][r[ix["Metric Name"]]] = float(r[ix["Metric Value"]].replace(",", ""))
    tot = collections.Counter()
    for v in per.values():
        tot.update(v)
    bench = None
    for line in open(log_path):
        if line.startswith("{") and '"metric"' in line:
            bench = json.loads(line)
    n = len(per)
    out = {"launches": n, "duration_ms": tot["gpu__time_duration.sum"] / 1e6,
           "pcie_read_bytes": tot["pcie__read_bytes.sum"], "pcie_write_bytes": tot["pcie__write_bytes.sum"],
           "dram_read_bytes": tot["dram__bytes_read.sum"], "dram_write_bytes": tot["dram__bytes_write.sum"],
           "per_launch": {"pcie_bytes": (tot["pcie__read_bytes.sum"] + tot["pcie__write_bytes.sum"]) / n,
                          "dram_bytes": (tot["dram__bytes_read.sum"] + tot["dram__bytes_write.sum"]) / n}}
    if bench:
        s = bench["stats_per_iter"]["eager"]
        link = s["h2d_bytes"] + s["d2h_bytes"]
        hbm = link + s["zf_bytes"]
        out["algorithmic"] = {"link_bytes": link, "hbm_bytes": hbm, "h2d_bytes": s["h2d_bytes"],
                              "d2h_bytes": s["d2h_bytes"], "zf_bytes": s["zf_bytes"],
                              "per_launch_link_bytes": link / n}
        out["ratio"] = {"pcie_over_link": (tot["pcie__read_bytes.sum"] + tot["pcie__write_bytes.sum"]) / link,
                        "pcie_write_over_d2h": tot["pcie__write_bytes.sum"] / s["d2h_bytes"] if s["d2h_bytes"] else None,
                        "pcie_read_over_h2d": tot["pcie__read_bytes.sum"] / s["h2d_bytes"] if s["h2d_bytes"] else None,
                        "dram_over_hbm": (tot["dram__bytes_read.sum"] + tot["dram__bytes_write.sum"]) / hbm}
        out["link_gbs_by_ncu_duration"] = link / (tot["gpu__time_duration.sum"] / 1e9) / 1e9
        out["bench_iter_ms_under_ncu"] = bench["ms_per_step"]
    print(json.dumps(out, indent=1))


if __name__ == "__main__":
    main(sys.argv[1], sys.argv[2])
