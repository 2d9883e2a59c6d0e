# round 2 (session 2): TMA gather4 ceiling; A/B of the warp-row pipeline / min-blocks knobs; plan's lane gather policy
mkdir -p gpurun_out /tmp/permcache
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r69_build.log 2>&1 || tail -20 gpurun_out/r69_build.log
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/gc scripts/gather_ceiling.cu -lcuda && timeout 300 /tmp/gc t > gpurun_out/r69_tma.jsonl 2> gpurun_out/r69_tma.err; echo "gc rc=$?"; cat gpurun_out/r69_tma.jsonl gpurun_out/r69_tma.err | cut -c1-200
for co in "5 rabbitpp" "3 rabbitpp"; do set -- $co
  it=""; [ "$1" = 5 ] && it="--iterate"
  for so in variants/head.so variants/p0m1.so variants/p1m1.so variants/p0m8.so paper_conf_ispass_balajicjk23_b200/libspmv.so; do
    timeout 1200 python scripts/kprof.py --config $1 --ordering $2 --steps 10 $it --so $so >> gpurun_out/r69_ab.jsonl 2>> gpurun_out/r69_ab.err
  done
done
for co in "4 rabbit" "4 rabbitpp" "2 rabbitpp" "1 rabbitpp"; do set -- $co
  for so in variants/head.so paper_conf_ispass_balajicjk23_b200/libspmv.so; do
    timeout 1200 python scripts/kprof.py --config $1 --ordering $2 --steps 10 --so $so >> gpurun_out/r69_ab.jsonl 2>> gpurun_out/r69_ab.err
  done
done
python - <<'PY'
import json
for l in open('gpurun_out/r69_ab.jsonl'):
    d=json.loads(l); print(d['workload'], d['ordering'], (d['so'] or '').split('/')[-1], 'cold', d['cold_ms'], 'warm', d['warm_ms'], 'it', d['iterate_ms'], d['x_ideal_cold'], d['y_sha'], d.get('lane_pred'), d.get('lane_waste'), d.get('lane_nnz'))
PY
