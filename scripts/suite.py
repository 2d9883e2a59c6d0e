"""C1-C5 suite on one B200 (north_star "geomean over the
synthetic suite"): runs bench.py once per BASELINE config with its paper
orderings, collects each JSON line and prints one summary line with the
geometric and arithmetic means of runtime / ideal (PAPER.md:120 reports means
without saying which; reading c24).

    python scripts/suite.py [--configs 1,2,3,4,5] [--out profiles/suite_r2.json]

Configs 1-4: one cold spmv_exec per step (L2 + persisting lines flushed);
config 5: one spmv_iterate power-iteration step (inputs >> L2).
"""
import argparse
import json
import math
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
ap = argparse.ArgumentParser()
ap.add_argument("--configs", default="1,2,3,4,5")
ap.add_argument("--steps", type=int, default=10)
ap.add_argument("--out", default=None)
ap.add_argument("--perm-cache", default="/tmp/permcache")
a = ap.parse_args()
orders = {1: "random,original,rabbit,rabbitpp", 2: "random,original,rabbit,rabbitpp",
          3: "random,original,rabbit,hubsort,rabbitpp", 4: "original,rabbit,rabbitpp",
          5: "original,rabbit,hubsort,rabbitpp"}
lines = []
for k in [int(c) for c in a.configs.split(",")]:
    cmd = [sys.executable, os.path.join(ROOT, "bench.py"), "--config", str(k), "--orderings",
           orders[k], "--steps", str(a.steps), "--warmup", "3", "--no-cpu-baseline",
           "--perm-cache", a.perm_cache]
    r = subprocess.run(cmd, capture_output=True, text=True, cwd=ROOT)
    out = [ln for ln in r.stdout.splitlines() if ln.startswith("{")]
    if r.returncode or not out:
        print(json.dumps({"config": k, "rc": r.returncode, "stderr": r.stderr[-2000:]}), flush=True)
        continue
    d = json.loads(out[-1])
    lines.append(d)
    print(json.dumps({"config": k, "workload": d["config"]["workload"],
                      "headline": d["config"]["ordering"], "ms": d["ms_per_step"],
                      "runtime_over_ideal": d["runtime_over_ideal"],
                      "orderings": {o: round(v["runtime_over_ideal"], 3)
                                    for o, v in d["orderings"].items()}}), flush=True)
r = [d["runtime_over_ideal"] for d in lines]
summary = {"suite": [d["config"]["workload"] for d in lines],
           "headline_runtime_over_ideal": r,
           "geomean": math.exp(sum(math.log(v) for v in r) / len(r)) if r else None,
           "mean": sum(r) / len(r) if r else None}
print(json.dumps(summary), flush=True)
if a.out:
    with open(a.out, "w") as f:
        json.dump({"summary": summary, "lines": lines}, f, indent=1)
