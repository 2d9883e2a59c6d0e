# round 2 (session 2): row-class kernels concurrent (3 streams, default) vs one stream, interleaved
mkdir -p gpurun_out /tmp/permcache
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r76_build.log 2>&1 || tail -20 gpurun_out/r76_build.log
for co in "5 rabbitpp" "3 rabbitpp"; do set -- $co
  it=""; [ "$1" = 5 ] && it="--iterate"
  for rep in 1 2; do
    for e in SPMV_CONCURRENT=1 SPMV_CONCURRENT=0; do
      timeout 1200 python scripts/kprof.py --config $1 --ordering $2 --steps 10 $it --env $e >> gpurun_out/r76_conc.jsonl 2>> gpurun_out/r76_conc.err
    done
  done
done
for rep in 1 2; do
  for e in SPMV_WIN_FRAC=0.5 SPMV_WIN_FRAC=0; do
    timeout 1200 python scripts/kprof.py --config 5 --ordering rabbitpp --steps 10 --iterate --env $e >> gpurun_out/r76_conc.jsonl 2>> gpurun_out/r76_conc.err
  done
done
python - <<'PY'
import json
for l in open('gpurun_out/r76_conc.jsonl'):
    d=json.loads(l); print(d['workload'], d['env'], 'cold', d['cold_ms'], 'warm', d['warm_ms'], 'scaled', d['scaled_fixed_ms'], 'it', d['iterate_ms'])
PY
for so in paper_conf_ispass_balajicjk23_b200/libspmv.so variants/ctapipe.so; do
  n=$(basename $so .so)
  timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --cache-control none --clock-control none -k regex:"k_lane|k_warp_rows|k_cta_rows|k_hub" --csv --log-file gpurun_out/r76_${n}.csv python scripts/kprof.py --config 5 --ordering rabbitpp --ncu 2 --so $so > /dev/null 2>&1; echo "ncu $n rc=$?"
done
