# round 2: L2 window size / hit ratio and MID stream-load mode across configs
mkdir -p gpurun_out /tmp/permcache
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r57_build.log 2>&1 || tail -20 gpurun_out/r57_build.log
run() { cfg=$1; ord=$2; shift 2; timeout 900 python scripts/kprof.py --config $cfg --ordering $ord --steps 8 --env "$@" >> gpurun_out/r57_knobs.log 2>> gpurun_out/r57_knobs.err; }
for cfg_ord in "5 rabbitpp" "5 hubsort" "3 rabbitpp" "4 rabbitpp" "2 rabbitpp"; do
  set -- $cfg_ord
  for kn in SPMV_NONE=1 SPMV_WIN_FRAC=0 SPMV_WIN_FRAC=0.16 SPMV_WIN_FRAC=0.25 SPMV_WIN_FRAC=0.33 SPMV_WIN_FRAC=0.5 SPMV_WIN_HIT=0.5 SPMV_MID_STREAM=1 SPMV_MID_STREAM=2; do
    run $1 $2 $kn
  done
  run $1 $2 SPMV_WIN_FRAC=0.33 SPMV_MID_STREAM=1
done
python - <<'PY'
import json
for l in open('gpurun_out/r57_knobs.log'):
    d = json.loads(l); print(d['workload'], d['ordering'], d['env'], d['cold_ms'], d['warm_ms'], d['x_ideal_cold'], d['win'], d['y_sha'])
PY
