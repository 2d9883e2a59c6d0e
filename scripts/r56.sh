# round 2: C5 RABBIT++ exec knobs (L2 window size, lane stream policy, entries in flight), ncu of k_warp_rows
mkdir -p gpurun_out /tmp/permcache
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r56_build.log 2>&1 || tail -20 gpurun_out/r56_build.log
run() { timeout 900 python scripts/kprof.py --config 5 --ordering rabbitpp --steps 8 --env "$@" >> gpurun_out/r56_knobs.log 2>> gpurun_out/r56_knobs.err; }
run SPMV_NONE=1
run SPMV_WIN_COLS=0
run SPMV_WIN_COLS=4194304
run SPMV_WIN_COLS=10485760
run SPMV_LANE_EF=1
run SPMV_LANE_EF=2
run SPMV_WARP_UNR=8
run SPMV_CTA_UNR=8
run SPMV_LANE_CTAS=8
run SPMV_FORK_EARLY=0
run SPMV_L2_FETCH=32
cat gpurun_out/r56_knobs.log | python -c "
import sys, json
for l in sys.stdin:
    d = json.loads(l); print(d['env'], d['cold_ms'], d['warm_ms'], d['x_ideal_cold'], d['win'], d['y_sha'])"
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:k_warp_rows -c 1 -o gpurun_out/r56_c5_warp_rows python scripts/kprof.py --config 5 --ordering rabbitpp --ncu 1 > gpurun_out/r56_ncu.log 2>&1; echo "ncu rc=$?"
for c in 2 3; do
  timeout 900 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum -k regex:"k_lane|k_warp_rows|k_cta_rows|k_hub" --csv --log-file gpurun_out/r56_fig6_c$c.csv python scripts/fig6.py --config $c --execs 2 >> gpurun_out/r56_fig6.log 2>&1
done
cat gpurun_out/r56_fig6.log | grep "{"
