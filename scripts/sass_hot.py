"""Top SASS instructions by executed count / stall samples from an ncu source-page CSV."""
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
h = rows[1]
ie, ss = h.index("Instructions Executed"), h.index("Warp Stall Sampling (All Samples)")
data = []
for r in rows[2:]:
    if len(r) < len(h):
        continue
    try:
        data.append((int(r[ie] or 0), int(r[ss] or 0), r[0], r[1]))
    except ValueError:
        pass
tot_i = sum(d[0] for d in data)
tot_s = sum(d[1] for d in data)
print("total instr", tot_i, "samples", tot_s)
key = 1 if len(sys.argv) > 2 and sys.argv[2] == "stall" else 0
for d in sorted(data, key=lambda d: -d[key])[:int(sys.argv[3]) if len(sys.argv) > 3 else 40]:
    print(f"{d[0]:>10} {100*d[0]/tot_i:5.1f}%  {d[1]:>6} {100*d[1]/max(tot_s,1):5.1f}%  {d[2]}  {d[3]}")
