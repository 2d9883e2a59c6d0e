# round 2 (session 2): A/B of the pipelined long-row sums (tree) and predicated lane gathers (pred) vs HEAD
mkdir -p gpurun_out /tmp/permcache
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r68_build.log 2>&1 || tail -20 gpurun_out/r68_build.log
for co in "1 rabbitpp" "2 rabbitpp" "3 rabbitpp" "4 rabbit" "5 rabbitpp"; do set -- $co
  it=""; [ "$1" = 5 ] && it="--iterate"
  for so in variants/head.so paper_conf_ispass_balajicjk23_b200/libspmv.so variants/pred.so; do
    timeout 1200 python scripts/kprof.py --config $1 --ordering $2 --steps 10 $it --so $so >> gpurun_out/r68_ab.jsonl 2>> gpurun_out/r68_ab.err
  done
done
for so in variants/su8.so variants/su16.so; do
  timeout 600 python scripts/kprof.py --config 1 --ordering rabbitpp --steps 20 --so $so >> gpurun_out/r68_ab.jsonl 2>> gpurun_out/r68_ab.err
done
python - <<'PY'
import json
for l in open('gpurun_out/r68_ab.jsonl'):
    d=json.loads(l); print(d['workload'], d['ordering'], (d['so'] or '').split('/')[-1], 'cold', d['cold_ms'], 'warm', d['warm_ms'], 'it', d['iterate_ms'], d['x_ideal_cold'], d['y_sha'])
PY
