# round 2 (session 2): targeted GPU tests of the new lane gather policy / k_small pipeline; C1/C4 timing;
# exec vs exec_scaled per-kernel launch list on C5 (where the power-iteration step's extra time goes);
# ncu --set full of k_lane on the stencil (predicated gathers)
mkdir -p gpurun_out /tmp/permcache
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r70_build.log 2>&1 || tail -20 gpurun_out/r70_build.log
timeout 1500 python -m pytest -q -m gpu tests/test_gpu_lane_pred.py tests/test_gpu_unroll.py tests/test_gpu_nonfinite.py "tests/test_gpu_parity.py::test_exec_matches_oracle" "tests/test_gpu_parity.py::test_small_plan_single_launch_bitwise" > gpurun_out/r70_tests.log 2>&1; echo "tests rc=$?"; tail -3 gpurun_out/r70_tests.log
for co in "1 rabbitpp" "4 rabbitpp"; do set -- $co
  timeout 900 python scripts/kprof.py --config $1 --ordering $2 --steps 20 >> gpurun_out/r70_kprof.jsonl 2>> gpurun_out/r70_kprof.err
done
cut -c1-400 gpurun_out/r70_kprof.jsonl
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct,launch__registers_per_thread,sm__warps_active.avg.pct_of_peak_sustained_active --cache-control none --clock-control none --csv --log-file gpurun_out/r70_c5_exec_vs_scaled.csv python scripts/kprof.py --config 5 --ordering rabbitpp --ncu 2 --ncu-scaled > gpurun_out/r70_ncu1.log 2>&1; echo "ncu1 rc=$?"
timeout 900 ncu --set full --import-source on --clock-control none -k regex:k_lane -s 1 -c 1 -o gpurun_out/r70_c4_klane python scripts/kprof.py --config 4 --ordering rabbitpp --ncu 2 > gpurun_out/r70_ncu2.log 2>&1; echo "ncu2 rc=$?"
