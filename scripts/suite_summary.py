"""Summarise a scripts/suite.sh run (bench lines + ncu exec-kernel metrics) into
profiles/suite_TAG.{json,md}.  Run here (no GPU):
    python scripts/suite_summary.py TAG
Per (config, ordering): bench cold / warm ms, runtime / ideal, and from ncu the
LAST exec's kernels (one launch each of k_lane / k_warp_rows / k_cta_rows /
k_hub_*): serialised time, DRAM bytes, DRAM / ideal, L2 hit per kernel."""
import collections
import csv
import glob
import io
import json
import os
import re
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
OUT = os.path.join(ROOT, "gpurun_out")
tag = sys.argv[1]
EXEC = ("k_lane", "k_warp_rows", "k_cta_rows", "k_hub_chunk", "k_hub_fix", "k_panel")


def ncu_last_exec(path):
    txt = open(path).read()
    i = txt.find('"ID"')
    if i < 0:
        return None
    rows = list(csv.DictReader(io.StringIO(txt[i:])))
    launches = collections.OrderedDict()
    for r in rows:
        k = (int(r["ID"]), r["Kernel Name"])
        launches.setdefault(k, {})[r["Metric Name"]] = float(r["Metric Value"].replace(",", ""))
    seq = [(re.search(r"::(k_\w+)", name).group(1), m) for (_, name), m in launches.items()
           if re.search(r"::(k_\w+)", name)]
    # the last exec = the last occurrence of each distinct kernel name
    last = {}
    for nm, m in seq:
        if nm in EXEC:
            last[nm] = m
    return last


res = {}
for jf in sorted(glob.glob(os.path.join(OUT, f"suite_{tag}_c*.json"))):
    cfg = re.search(r"_c(\d+)\.json", jf).group(1)
    txt = open(jf).read().strip()
    if not txt:
        continue
    d = json.loads(txt.splitlines()[-1])
    ideal = d["config"]["ideal_bytes"]
    for o, v in d["orderings"].items():
        e = {"workload": d["config"]["workload"], "n": d["config"]["n"], "nnz": d["config"]["nnz"],
             "ideal_bytes": ideal, "ms_cold": v["ms"], "ms_warm": v["warm_ms"],
             "runtime_over_ideal": v["runtime_over_ideal"], "reorder_s": v["reorder_s"],
             "insularity": v["insularity"], "H": v["H"], "l2_window_bytes": v["l2_window_bytes"],
             "gflops": v["gflops"]}
        for side in ("spmm4", "coo"):
            if side in v:
                e[side] = v[side]
        nf = os.path.join(OUT, f"suite_{tag}_c{cfg}_{o}_ncu.csv")
        if os.path.exists(nf):
            last = ncu_last_exec(nf)
            if last:
                dram = sum(m.get("dram__bytes_read.sum", 0) + m.get("dram__bytes_write.sum", 0)
                           for m in last.values())
                e["ncu"] = {k: {"us": round(m.get("gpu__time_duration.sum", 0) / 1e3, 1),
                                "dram_bytes": m.get("dram__bytes_read.sum", 0) + m.get("dram__bytes_write.sum", 0),
                                "l2_hit_pct": m.get("lts__t_sector_hit_rate.pct")}
                            for k, m in last.items()}
                e["dram_bytes"] = dram
                e["dram_over_ideal"] = round(dram / ideal, 4)
                e["ncu_serial_ms"] = round(sum(m.get("gpu__time_duration.sum", 0) for m in last.values()) / 1e6, 4)
        res[f"c{cfg}/{o}"] = e
os.makedirs(os.path.join(ROOT, "profiles"), exist_ok=True)
json.dump(res, open(os.path.join(ROOT, "profiles", f"suite_{tag}.json"), "w"), indent=1)
lines = [f"| config/ordering | ms cold | ms warm | x ideal | DRAM / ideal | ncu serial ms | kernels (us, DRAM GB, L2 hit %) |",
         "|---|---|---|---|---|---|---|"]
for k, e in res.items():
    ks = "; ".join(f"{n} {m['us']}, {m['dram_bytes'] / 1e9:.2f}, {m['l2_hit_pct']}" for n, m in e.get("ncu", {}).items())
    lines.append(f"| {k} | {e['ms_cold']:.4f} | {e['ms_warm']:.4f} | {e['runtime_over_ideal']:.3f} | "
                 f"{e.get('dram_over_ideal', '—')} | {e.get('ncu_serial_ms', '—')} | {ks} |")
md = "\n".join(lines)
open(os.path.join(ROOT, "profiles", f"suite_{tag}.md"), "w").write(md + "\n")
print(md)
