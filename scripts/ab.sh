# A/B of libspmv builds or dev knobs under gpurun, one cached permutation per
# config so the arms see the same matrix (the concurrent RABBIT detection gives
# a different permutation each run):
#   python scripts/variant.py --rev HEAD --out variants/head.so      (here)
#   gpurun -- 'bash scripts/ab.sh "5:rabbitpp 3:rabbitpp" "variants/head.so paper_conf_ispass_balajicjk23_b200/libspmv.so" [ENV=VAL ...]'
# Each (config, build) runs twice, interleaved; kprof prints cold / warm /
# exec_scaled / iterate times and y's hash (bitwise check across arms).
SPECS=$1; SOS=$2; shift 2
mkdir -p gpurun_out /tmp/permcache
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/ab_build.log 2>&1 || tail -20 gpurun_out/ab_build.log
for spec in $SPECS; do
  cfg=${spec%%:*}; ord=${spec#*:}; it=""; [ "$cfg" = 5 ] && it="--iterate"
  for rep in 1 2; do
    for so in $SOS; do
      timeout 1200 python scripts/kprof.py --config $cfg --ordering $ord --steps 10 $it --so $so --env "$@" >> gpurun_out/ab.jsonl 2>> gpurun_out/ab.err
    done
  done
done
python - <<'PY'
import json
for l in open('gpurun_out/ab.jsonl'):
    d=json.loads(l); print(d['workload'], d['ordering'], (d['so'] or '').split('/')[-1], d['env'], 'cold', d['cold_ms'], 'warm', d['warm_ms'], 'scaled', d['scaled_fixed_ms'], 'it', d['iterate_ms'], d['y_sha'])
PY
