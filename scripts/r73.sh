# round 2 (session 2): norm from y (no per-row partial stores), register CTA sorts in P A P^T,
# full GPU suite, C5 iterate A/B vs HEAD (same process order), permute timing, exec vs scaled launch list
mkdir -p gpurun_out /tmp/permcache
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r73_build.log 2>&1 || tail -20 gpurun_out/r73_build.log
timeout 2400 python -m pytest tests -q -m gpu -x > gpurun_out/r73_tests.log 2>&1; echo "tests rc=$?"; tail -5 gpurun_out/r73_tests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
for co in "5 rabbitpp" "3 rabbitpp"; do set -- $co
  it=""; [ "$1" = 5 ] && it="--iterate"
  for so in variants/head.so paper_conf_ispass_balajicjk23_b200/libspmv.so variants/head.so paper_conf_ispass_balajicjk23_b200/libspmv.so; do
    timeout 1200 python scripts/kprof.py --config $1 --ordering $2 --steps 10 $it --so $so >> gpurun_out/r73_ab.jsonl 2>> gpurun_out/r73_ab.err
  done
done
python - <<'PY'
import json
for l in open('gpurun_out/r73_ab.jsonl'):
    d=json.loads(l); print(d['workload'], d['ordering'], (d['so'] or '').split('/')[-1], 'cold', d['cold_ms'], 'warm', d['warm_ms'], 'scaled', d['scaled_fixed_ms'], 'it', d['iterate_ms'], d['y_sha'], 'permute_ms', d.get('permute_ms'))
PY
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct --cache-control none --clock-control none --csv --log-file gpurun_out/r73_c5_exec_vs_scaled.csv python scripts/kprof.py --config 5 --ordering rabbitpp --ncu 2 --ncu-scaled > gpurun_out/r73_ncu1.log 2>&1; echo "ncu1 rc=$?"
