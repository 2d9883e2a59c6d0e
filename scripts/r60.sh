# round 2: C2 A/B against the round-1 tree on the same box, then the C1-C5 suite -> profiles
mkdir -p gpurun_out /tmp/permcache
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r60_build.log 2>&1 || tail -20 gpurun_out/r60_build.log
(cd scratch_old && python -c "import __graft_entry__ as g; g.build()" > ../gpurun_out/r60_old_build.log 2>&1 && \
  timeout 600 python bench.py --config 2 --orderings rabbit,rabbitpp --steps 30 --warmup 5 --no-cpu-baseline --no-side > ../gpurun_out/r60_old_c2.json 2>/dev/null)
timeout 600 python bench.py --config 2 --orderings rabbit,rabbitpp --steps 30 --warmup 5 --no-cpu-baseline --no-side > gpurun_out/r60_new_c2.json 2>/dev/null
python - <<'PY'
import json
for t in ("old", "new"):
    d = json.loads(open(f"gpurun_out/r60_{t}_c2.json").read())
    print(t, {k: round(v["ms"], 5) for k, v in d["orderings"].items()}, d.get("clocks"))
PY
SPMV_REORDER_VERBOSE=1 timeout 5000 python scripts/suite.py --configs 1,2,3,4,5 --steps 10 --out gpurun_out/suite_r60.json 2> gpurun_out/r60_suite.err | tee gpurun_out/r60_suite.log
