# round 2 (session 2): fresh-box check of the tree + random-gather ceilings
mkdir -p gpurun_out /tmp/permcache
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r67_build.log 2>&1 || tail -20 gpurun_out/r67_build.log
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/gc scripts/gather_ceiling.cu -lcuda && timeout 300 /tmp/gc > gpurun_out/r67_gather.jsonl 2> gpurun_out/r67_gather.err; echo "gc rc=$?"; cat gpurun_out/r67_gather.jsonl | cut -c1-200
timeout 2400 python -m pytest tests -q -m gpu > gpurun_out/r67_tests.log 2>&1; echo "tests rc=$?"; tail -3 gpurun_out/r67_tests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
SPMV_REORDER_VERBOSE=1 timeout 1800 python bench.py --steps 20 --warmup 5 > gpurun_out/r67_bench.json 2> gpurun_out/r67_bench.err; echo "bench rc=$?"
python -c "
import json;d=json.loads(open('gpurun_out/r67_bench.json').read())
print(d['value'], d['ms_per_step'], d['runtime_over_ideal'], d['roofline']['frac'], d['gpu_launches'], d['clocks'], d['input_prep'])
print(d['e2e'])
for k,v in d['orderings'].items(): print(k, {kk: v[kk] for kk in ('ms','runtime_over_ideal','reorder_s','permute_ms','permute_gbs','H','l2_window_bytes') if kk in v})
print(d.get('cpu_baseline'))"
timeout 1200 python bench.py --impl reference --steps 5 --warmup 3 > gpurun_out/r67_ref.json 2> gpurun_out/r67_ref.err; echo "ref rc=$?"; cut -c1-400 gpurun_out/r67_ref.json
timeout 1800 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct --clock-control none --csv --log-file gpurun_out/r67_launches.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-side --perm-cache /tmp/permcache --orderings rabbitpp > gpurun_out/r67_ncu_bench.log 2>&1; echo "ncu rc=$?"; wc -l gpurun_out/r67_launches.csv
