"""Update profiles/ncu_summary.json["kron28/rabbitpp"] (read by bench.py for
roofline.traffic) from an ncu launch list of the bench step (`ncu --metrics
gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum ...
--cache-control none --csv`): the last complete launch sequence of one step.

    python scripts/update_ncu_summary.py gpurun_out/r75_launches.csv TAG
"""
import collections
import csv
import json
import os
import re
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
STEP = ["k_lane", "k_warp_rows", "k_cta_rows", "k_hub_chunk", "k_hub_fix", "k_ss_y", "k_ss_final"]
rows = list(csv.reader(open(sys.argv[1])))
tag = sys.argv[2]
hi = [i for i, r in enumerate(rows) if "Kernel Name" in r][0]
h = rows[hi]
ki, mi, vi, idi = h.index("Kernel Name"), h.index("Metric Name"), h.index("Metric Value"), h.index("ID")
per, names = collections.defaultdict(dict), {}
for r in rows[hi + 1:]:
    if len(r) <= vi:
        continue
    per[int(r[idi])][r[mi]] = float(r[vi].replace(",", ""))
    n = re.sub(r"\(.*", "", r[ki].replace("(anonymous namespace)::", "").replace("spmv::", ""))
    names[int(r[idi])] = re.sub(r"<.*", "", n.replace("void ", "").replace("<unnamed>::", "")).strip()
ids = sorted(per)
# last index of k_ss_final, then walk back to the preceding k_lane
end = max(i for i in ids if names[i] == "k_ss_final")
start = max(i for i in ids if i < end and names[i] == "k_lane")
step = [i for i in ids if start <= i <= end and names[i] in STEP]
pk_us = collections.defaultdict(float)
pk_gb = collections.defaultdict(float)
dram = dread = dwrite = 0.0
for i in step:
    d = per[i]
    pk_us[names[i]] += d.get("gpu__time_duration.sum", 0) / 1e3
    b = d.get("dram__bytes_read.sum", 0) + d.get("dram__bytes_write.sum", 0)
    pk_gb[names[i]] += b / 1e9
    dram += b
    dread += d.get("dram__bytes_read.sum", 0)
    dwrite += d.get("dram__bytes_write.sum", 0)
p = os.path.join(ROOT, "profiles", "ncu_summary.json")
js = json.load(open(p))
js["kron28/rabbitpp"] = {
    "dram_bytes": dram, "dram_read": dread, "dram_write": dwrite,
    "duration_us": round(sum(pk_us.values()), 1),
    "kernel": "one power-iteration step (spmv_iterate): " + " + ".join(STEP) + " (serialised under ncu, "
              "--cache-control none)",
    "per_kernel_us": {k: round(v, 1) for k, v in pk_us.items()},
    "per_kernel_dram_gb": {k: round(v, 2) for k, v in pk_gb.items()},
    "source": sys.argv[1].replace("gpurun_out", "profiles"), "tag": tag}
json.dump(js, open(p, "w"), indent=1)
print(json.dumps(js["kron28/rabbitpp"], indent=1))
