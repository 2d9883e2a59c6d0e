# round 2: fresh-box check of the tree: full GPU suite, smoke, default bench (C5), reference arm,
# C2 bench, coop retry, ncu launch list of the default bench
mkdir -p gpurun_out /tmp/permcache
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r59_build.log 2>&1 || tail -20 gpurun_out/r59_build.log
timeout 2400 python -m pytest tests -q -m gpu > gpurun_out/r59_tests.log 2>&1; echo "tests rc=$?"; tail -3 gpurun_out/r59_tests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
SPMV_REORDER_VERBOSE=1 timeout 1800 python bench.py --steps 20 --warmup 5 > gpurun_out/r59_bench.json 2> gpurun_out/r59_bench.err; echo "bench rc=$?"
python -c "
import json;d=json.loads(open('gpurun_out/r59_bench.json').read())
print(d['value'], d['ms_per_step'], d['runtime_over_ideal'], d['roofline']['frac'], d['gpu_launches'], d['clocks'], d['input_prep'])
print(d['e2e'])
for k,v in d['orderings'].items(): print(k, {kk: v[kk] for kk in ('ms','runtime_over_ideal','reorder_s','permute_ms','permute_gbs','H','l2_window_bytes') if kk in v})
print(d.get('cpu_baseline')); print({k: d[k] for k in d if k.startswith('amort')})"
grep "spmv_reorder\]" gpurun_out/r59_bench.err | tail -12
timeout 1200 python bench.py --impl reference --steps 5 --warmup 3 > gpurun_out/r59_ref.json 2> gpurun_out/r59_ref.err; echo "ref rc=$?"; cut -c1-400 gpurun_out/r59_ref.json
timeout 900 python bench.py --config 2 --steps 20 --warmup 5 --no-cpu-baseline > gpurun_out/r59_bench_c2.json 2> gpurun_out/r59_bench_c2.err; echo "c2 rc=$?"
python -c "
import json;d=json.loads(open('gpurun_out/r59_bench_c2.json').read())
for k,v in d['orderings'].items(): print(k, {kk: v[kk] for kk in ('ms','runtime_over_ideal','permute_ms','permute_gbs') if kk in v})"
for co in "4 rabbit" "5 rabbitpp"; do set -- $co
  timeout 900 python scripts/kprof.py --config $1 --ordering $2 --steps 10 --env SPMV_LANE_COOP=1 >> gpurun_out/r59_coop.log 2>> gpurun_out/r59_coop.err
done; cat gpurun_out/r59_coop.log
timeout 1800 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r59_launches.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-side --perm-cache /tmp/permcache --orderings rabbitpp > gpurun_out/r59_ncu_bench.log 2>&1; echo "ncu rc=$?"; wc -l gpurun_out/r59_launches.csv
