# round 2 (session 2): fresh-box check of the final tree: full GPU suite, smoke, default bench (C5),
# reference arm, ncu launch list of the bench step (cache control none: DRAM bytes per step as run),
# ncu --set full of the top kernel (k_warp_rows, C5 RABBIT++)
mkdir -p gpurun_out /tmp/permcache
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r75_build.log 2>&1 || tail -20 gpurun_out/r75_build.log
timeout 2400 python -m pytest tests -q -m gpu > gpurun_out/r75_tests.log 2>&1; echo "tests rc=$?"; tail -3 gpurun_out/r75_tests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
SPMV_REORDER_VERBOSE=1 timeout 2400 python bench.py --steps 20 --warmup 5 > gpurun_out/r75_bench.json 2> gpurun_out/r75_bench.err; echo "bench rc=$?"
python -c "
import json;d=json.loads(open('gpurun_out/r75_bench.json').read())
print(d['value'], d['ms_per_step'], d['runtime_over_ideal'], d['roofline']['frac'], d.get('gather_roofline'), d['gpu_launches'], d['clocks'], d['input_prep'])
print(d['e2e'])
for k,v in d['orderings'].items(): print(k, {kk: v[kk] for kk in ('ms','runtime_over_ideal','reorder_s','permute_ms','permute_gbs','H','l2_window_bytes') if kk in v})
print(d.get('cpu_baseline'))"
timeout 1200 python bench.py --impl reference --steps 5 --warmup 3 > gpurun_out/r75_ref.json 2> gpurun_out/r75_ref.err; echo "ref rc=$?"; cut -c1-300 gpurun_out/r75_ref.json
timeout 1800 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct --cache-control none --clock-control none --csv --log-file gpurun_out/r75_launches.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-side --perm-cache /tmp/permcache --orderings rabbitpp > gpurun_out/r75_ncu_bench.log 2>&1; echo "ncu rc=$?"; wc -l gpurun_out/r75_launches.csv
timeout 1200 ncu --set full --import-source on --clock-control none -k regex:k_warp_rows -s 1 -c 1 -o gpurun_out/r75_c5_warp_rows python scripts/kprof.py --config 5 --ordering rabbitpp --ncu 2 > gpurun_out/r75_ncu2.log 2>&1; echo "ncu2 rc=$?"
