"""Dev: per-launch table from an `ncu --csv --metrics ...` log (kernel, time, DRAM GB, other metrics)."""
import collections
import csv
import re
import sys

rows = list(csv.reader(open(sys.argv[1])))
hi = [i for i, r in enumerate(rows) if "Kernel Name" in r][0]
h = rows[hi]
ki, mi, vi, idi = h.index("Kernel Name"), h.index("Metric Name"), h.index("Metric Value"), h.index("ID")
per, names = collections.defaultdict(dict), {}
for r in rows[hi + 1:]:
    if len(r) <= vi:
        continue
    try:
        per[r[idi]][r[mi]] = float(r[vi].replace(",", ""))
    except ValueError:
        continue
    n = r[ki].replace("(anonymous namespace)::", "").replace("spmv::", "")
    names[r[idi]] = re.sub(r"\(.*", "", n).replace("void ", "")
skip = int(sys.argv[2]) if len(sys.argv) > 2 else 0
for i in sorted(per, key=int)[skip:]:
    d = per[i]
    t = d.get("gpu__time_duration.sum", 0) / 1e3
    dram = (d.get("dram__bytes_read.sum", 0) + d.get("dram__bytes_write.sum", 0)) / 1e9
    extra = {k.split("__")[1][:24]: round(v, 2) for k, v in d.items()
             if k not in ("gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum")}
    print(f"{i:>5} {names[i][:48]:<48} {t:10.3f} us->ms? {t/1e3:9.3f} ms {dram:8.2f} GB {extra}")
