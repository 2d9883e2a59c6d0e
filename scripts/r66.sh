# round 2: where the power-iteration step's extra ~2 ms over the exec goes (C5 RABBIT++)
mkdir -p gpurun_out /tmp/permcache
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r66_build.log 2>&1 || tail -20 gpurun_out/r66_build.log
for e in SPMV_NONE=1 SPMV_WIN_FRAC=0 SPMV_CONCURRENT=0; do
  timeout 900 python scripts/kprof.py --config 5 --ordering rabbitpp --steps 10 --iterate --env $e 2>>gpurun_out/r66.err | python -c "import sys,json; d=json.loads(sys.stdin.read()); print(d['env'], 'cold', d['cold_ms'], 'warm', d['warm_ms'], 'scaled_fixed', d['scaled_fixed_ms'], 'iterate', d['iterate_ms'], d['win'])"
done
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct --clock-control none --csv --log-file gpurun_out/r66_iter_ncu.csv python scripts/kprof.py --config 5 --ordering rabbitpp --steps 2 --iterate > gpurun_out/r66_ncu.log 2>&1; echo "ncu rc=$?"
