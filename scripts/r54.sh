# round 2: C5 reorder at scale (time, memory), kernel times per ordering, launch list, bench
mkdir -p gpurun_out /tmp/permcache
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r54_build.log 2>&1 || tail -20 gpurun_out/r54_build.log
for o in original rabbitpp; do
  SPMV_REORDER_VERBOSE=1 timeout 1200 python scripts/kprof.py --config 5 --ordering $o --steps 10 --iterate >> gpurun_out/r54_kprof.log 2>> gpurun_out/r54_kprof.err
  echo "kprof $o rc=$?"
done
cat gpurun_out/r54_kprof.log; grep spmv_reorder gpurun_out/r54_kprof.err | tail -12
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct,l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum,l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum --clock-control none --csv --log-file gpurun_out/r54_c5_rabbitpp_ncu.csv python scripts/kprof.py --config 5 --ordering rabbitpp --ncu 1 > gpurun_out/r54_ncu.log 2>&1; echo "ncu rc=$?"
python - <<'PY'
import csv, collections
rows = list(csv.reader(open('gpurun_out/r54_c5_rabbitpp_ncu.csv')))
hdr = next(i for i, r in enumerate(rows) if r and r[0] == 'ID')
H = rows[hdr]; d = collections.OrderedDict()
for r in rows[hdr + 1:]:
    if len(r) < len(H): continue
    k = (r[H.index('ID')], r[H.index('Kernel Name')][:40]); d.setdefault(k, {})[r[H.index('Metric Name')]] = r[H.index('Metric Value')]
for k, v in list(d.items())[-12:]: print(k, v)
PY
SPMV_REORDER_VERBOSE=1 timeout 1500 python bench.py --steps 20 --warmup 5 > gpurun_out/r54_bench.json 2> gpurun_out/r54_bench.err; echo "bench rc=$?"; grep -v "^$" gpurun_out/r54_bench.err | tail -12
python -c "
import json;d=json.loads(open('gpurun_out/r54_bench.json').read())
print(d['value'], d['ms_per_step'], d['runtime_over_ideal'], d['roofline']['frac'], d['e2e'], d['gpu_launches'], d['clocks'], d['input_prep'])
for k,v in d['orderings'].items(): print(k, v)
print(d.get('cpu_baseline'))"
