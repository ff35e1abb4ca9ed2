#!/usr/bin/env python3
"""Summarise scripts/ncu_rank.sh CSVs into achieved NVLink / PCIe GB/s per kernel
against 900 GB/s NVLink 5 per direction and 64 GB/s PCIe Gen5 x16 (north star), and
write profiles/ncu_nvlink.json (bench.py's N > 1 roofline.traffic).

    python scripts/nvlink_summary.py <dir with ncu_rank*.csv> <world> <bytes> [--out profiles/ncu_nvlink.json]
"""
import csv
import glob
import json
import os
import sys
from collections import defaultdict


def rows(path):
    with open(path) as f:
        lines = [ln for ln in f if ln.startswith('"')]
    return list(csv.DictReader(lines))


def main():
    d, world, n = sys.argv[1], int(sys.argv[2]), int(sys.argv[3])
    out = sys.argv[sys.argv.index("--out") + 1] if "--out" in sys.argv else "profiles/ncu_nvlink.json"
    per = defaultdict(lambda: defaultdict(list))
    for p in sorted(glob.glob(os.path.join(d, "ncu_rank*.csv"))):
        rank = int(os.path.basename(p)[8:-4])
        for r in rows(p):
            # "void mpx::<unnamed>::send_kernel<6>(mpx::SendParams)" -> "send_kernel"
            k = r["Kernel Name"].split("(")[0].split("::")[-1].split("<")[0]
            try:
                v = float(r["Metric Value"].replace(",", ""))
            except ValueError:
                continue
            per[(rank, k)][r["Metric Name"]].append(v)
    summary = {}
    for (rank, k), m in sorted(per.items()):
        t = m.get("gpu__time_duration.sum", [0])
        launches = len(t)
        ts = sum(t) * 1e-9 if t else 0.0
        def gbs(name):
            return sum(m.get(name, [0])) / ts / 1e9 if ts else None
        summary[f"rank{rank}:{k}"] = {
            "launches": launches, "avg_us": ts / max(1, launches) * 1e6,
            "nvlink_tx_GBps": gbs("nvltx__bytes_data_user.sum"), "nvlink_rx_GBps": gbs("nvlrx__bytes_data_user.sum"),
            "pcie_read_GBps": gbs("pcie__read_bytes.sum"), "pcie_write_GBps": gbs("pcie__write_bytes.sum"),
            "nvlink_tx_bytes_per_launch": sum(m.get("nvltx__bytes_data_user.sum", [0])) / max(1, launches),
            "frac_tx_of_900": (gbs("nvltx__bytes_data_user.sum") or 0) / 900.0}
    doc = json.load(open(out)) if os.path.exists(out) else {}
    doc[f"{world}:{n}"] = summary
    with open(out, "w") as f:
        json.dump(doc, f, indent=1)
    print(json.dumps(summary, indent=1))


if __name__ == "__main__":
    main()
