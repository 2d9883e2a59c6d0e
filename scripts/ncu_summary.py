"""Summarise ncu captures into profiles/ (run here, no GPU needed).

    python scripts/ncu_summary.py TAG WORKLOAD gpurun_out/prof_TAG_rabbitpp.ncu-rep[:ordering] ...
    python scripts/ncu_summary.py --launches gpurun_out/launches_TAG.csv

Writes/updates profiles/ncu_summary.json (keyed "workload/ordering", read by
bench.py for roofline.traffic) and prints a markdown table.
"""
from __future__ import annotations

import csv
import io
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
KEYS = {
    "gpu__time_duration.sum": "duration_us",
    "dram__bytes_read.sum": "dram_read",
    "dram__bytes_write.sum": "dram_write",
    "lts__t_sector_hit_rate.pct": "l2_hit_pct",
    "l1tex__t_sector_hit_rate.pct": "l1_hit_pct",
    "dram__throughput.avg.pct_of_peak_sustained_elapsed": "dram_pct_peak",
    "sm__warps_active.avg.pct_of_peak_sustained_active": "occupancy_pct",
    "smsp__average_warps_issue_stalled_long_scoreboard_per_issue_active.ratio": "stall_long_sb",
    "smsp__average_warp_latency_per_inst_issued.ratio": "cycles_per_issue",
    "launch__registers_per_thread": "regs",
    "launch__grid_size": "grid",
}
UNIT = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "usecond": 1, "msecond": 1e3,
        "nsecond": 1e-3}


def raw(rep: str):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True,
                         text=True, check=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr, units, data = rows[0], rows[1], rows[2:]
    res = []
    for d in data:
        e = {"kernel": d[hdr.index("Kernel Name")]}
        for k, nm in KEYS.items():
            if k in hdr:
                i = hdr.index(k)
                v = d[i].replace(",", "")
                try:
                    f = float(v)
                except ValueError:
                    continue
                f *= UNIT.get(units[i], 1)
                e[nm] = f
        if "dram_read" in e:
            e["dram_bytes"] = e["dram_read"] + e.get("dram_write", 0)
        res.append(e)
    return res


def launches(path: str):
    rows = list(csv.reader(open(path)))
    hdr = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
    h = rows[hdr]
    tot = {}
    for r in rows[hdr + 1:]:
        if len(r) < len(h) or r[h.index("Metric Name")] != "gpu__time_duration.sum":
            continue
        k = r[h.index("Kernel Name")].replace("void ", "").replace("<unnamed>::", "")
        k = k.replace("(anonymous namespace)::", "").split("(")[0]
        v = float(r[h.index("Metric Value")].replace(",", ""))
        u = r[h.index("Metric Unit")]
        v *= {"nsecond": 1e-3, "ns": 1e-3, "usecond": 1, "us": 1, "msecond": 1e3, "ms": 1e3}.get(u, 1)
        t = tot.setdefault(k, [0, 0.0])
        t[0] += 1
        t[1] += v
    return tot


def main():
    if sys.argv[1] == "--launches":
        tot = launches(sys.argv[2])
        s = sum(v[1] for v in tot.values())
        print("| kernel | launches | total us | share |\n|---|---|---|---|")
        for k, (n, us) in sorted(tot.items(), key=lambda kv: -kv[1][1]):
            print(f"| {k} | {n} | {us:.1f} | {100 * us / s:.1f}% |")
        return
    tag, workload = sys.argv[1], sys.argv[2]
    path = os.path.join(ROOT, "profiles", "ncu_summary.json")
    summ = json.load(open(path)) if os.path.exists(path) else {}
    print("| workload/ordering | kernel | us | DRAM bytes | L2 hit % | L1 hit % | DRAM % peak | occ % |")
    print("|---|---|---|---|---|---|---|---|")
    for arg in sys.argv[3:]:
        rep, _, ordering = arg.partition(":")
        for e in raw(rep):
            e["tag"] = tag
            e["source"] = os.path.basename(rep)
            summ[f"{workload}/{ordering}"] = e
            print(f"| {workload}/{ordering} | {e['kernel'][:40]} | {e.get('duration_us', 0):.1f} | "
                  f"{e.get('dram_bytes', 0):.4g} | {e.get('l2_hit_pct', 0):.1f} | "
                  f"{e.get('l1_hit_pct', 0):.1f} | {e.get('dram_pct_peak', 0):.1f} | "
                  f"{e.get('occupancy_pct', 0):.1f} |")
    os.makedirs(os.path.dirname(path), exist_ok=True)
    json.dump(summ, open(path, "w"), indent=1, sort_keys=True)


if __name__ == "__main__":
    main()
