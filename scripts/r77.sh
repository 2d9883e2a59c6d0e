# round 2 (session 2): k_lane chunks in flight (unroll 1 / 2 / 4) on the stencil and SBM (serialised ncu time + cold events)
mkdir -p gpurun_out /tmp/permcache
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r77_build.log 2>&1 || tail -20 gpurun_out/r77_build.log
for co in "4 rabbitpp" "2 rabbitpp"; do set -- $co
  for so in variants/lu1.so paper_conf_ispass_balajicjk23_b200/libspmv.so variants/lu4.so; do
    timeout 900 python scripts/kprof.py --config $1 --ordering $2 --steps 10 --so $so >> gpurun_out/r77_ab.jsonl 2>> gpurun_out/r77_ab.err
    n=$(basename $so .so)
    timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,launch__registers_per_thread --clock-control none -k regex:"k_lane" --csv --log-file gpurun_out/r77_c$1_${n}.csv python scripts/kprof.py --config $1 --ordering $2 --ncu 3 --so $so > /dev/null 2>&1
  done
done
python - <<'PY'
import json
for l in open('gpurun_out/r77_ab.jsonl'):
    d=json.loads(l); print(d['workload'], (d['so'] or '').split('/')[-1], 'cold', d['cold_ms'], 'warm', d['warm_ms'], d['y_sha'])
PY
for f in gpurun_out/r77_c*.csv; do echo $f; python scripts/ncu_list.py $f | tail -3 | cut -c1-160; done
