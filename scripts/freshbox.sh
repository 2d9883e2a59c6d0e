# Fresh-box check under gpurun (one parametrised script for every round's
# end-of-work call; the per-call launchers r31..r77 were folded into this):
#   /usr/local/graft/bin/gpurun --timeout 5400 -- 'bash scripts/freshbox.sh TAG'
# full GPU suite, smoke, default bench (C5 power iteration), reference arm,
# ncu launch list of the bench step (DRAM bytes per step as run: cache control
# none), ncu --set full of the top kernel (k_warp_rows on C5 RABBIT++).
# Outputs gpurun_out/TAG_*; summarise with scripts/update_ncu_summary.py.
TAG=${1:-check}
mkdir -p gpurun_out /tmp/permcache
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/${TAG}_build.log 2>&1 || tail -20 gpurun_out/${TAG}_build.log
timeout 2400 python -m pytest tests -q -m gpu > gpurun_out/${TAG}_tests.log 2>&1; echo "tests rc=$?"; tail -3 gpurun_out/${TAG}_tests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
[ -n "$SKIP_BENCH" ] && exit 0
SPMV_REORDER_VERBOSE=1 timeout 2400 python bench.py --steps 20 --warmup 5 > gpurun_out/${TAG}_bench.json 2> gpurun_out/${TAG}_bench.err; echo "bench rc=$?"
python -c "
import json;d=json.loads(open('gpurun_out/${TAG}_bench.json').read())
print(d['value'], d['ms_per_step'], d['runtime_over_ideal'], d['roofline']['frac'], d.get('gather_roofline'), d['gpu_launches'], d['clocks'], d['input_prep'])
print(d['e2e'])
for k,v in d['orderings'].items(): print(k, {kk: v[kk] for kk in ('ms','runtime_over_ideal','reorder_s','permute_ms','permute_gbs','H','l2_window_bytes') if kk in v})
print(d.get('cpu_baseline'))"
timeout 1200 python bench.py --impl reference --steps 5 --warmup 3 > gpurun_out/${TAG}_ref.json 2> gpurun_out/${TAG}_ref.err; echo "ref rc=$?"; cut -c1-300 gpurun_out/${TAG}_ref.json
[ -n "$SKIP_NCU" ] && exit 0
timeout 1800 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct --cache-control none --clock-control none --csv --log-file gpurun_out/${TAG}_launches.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-side --perm-cache /tmp/permcache --orderings rabbitpp > gpurun_out/${TAG}_ncu_bench.log 2>&1; echo "ncu rc=$?"; wc -l gpurun_out/${TAG}_launches.csv
timeout 1200 ncu --set full --import-source on --clock-control none -k regex:k_warp_rows -s 1 -c 1 -o gpurun_out/${TAG}_c5_warp_rows python scripts/kprof.py --config 5 --ordering rabbitpp --ncu 2 > gpurun_out/${TAG}_ncu2.log 2>&1; echo "ncu2 rc=$?"
