# round 2: tests of the new kernels / gates, then k_lane_coop, k_small and the flush reset measured
mkdir -p gpurun_out /tmp/permcache
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r58_build.log 2>&1 || tail -20 gpurun_out/r58_build.log
timeout 1500 python -m pytest -q -m gpu -x tests/test_gpu_unroll.py tests/test_gpu_nccl_iterate.py "tests/test_gpu_parity.py::test_small_plan_single_launch_bitwise" "tests/test_gpu_parity.py::test_hot_prefix_window_gate" "tests/test_gpu_parity.py::test_permute_and_bins_bitexact" "tests/test_gpu_parity.py::test_exec_matches_oracle" > gpurun_out/r58_tests.log 2>&1; echo "tests rc=$?"; tail -5 gpurun_out/r58_tests.log
run() { cfg=$1; ord=$2; shift 2; timeout 900 python scripts/kprof.py --config $cfg --ordering $ord --steps 10 "$@" >> gpurun_out/r58_knobs.log 2>> gpurun_out/r58_knobs.err; }
run 2 rabbitpp --env SPMV_NONE=1
run 2 rabbitpp --no-reset --env SPMV_NONE=1
run 1 rabbitpp --env SPMV_SMALL=0
run 1 rabbitpp --env SPMV_SMALL=1
for co in "4 rabbit" "4 planted" "3 rabbitpp" "5 rabbitpp"; do
  set -- $co
  run $1 $2 --env SPMV_LANE_COOP=0
  run $1 $2 --env SPMV_LANE_COOP=1
done
python - <<'PY'
import json
for l in open('gpurun_out/r58_knobs.log'):
    d = json.loads(l); print(d['workload'], d['ordering'], d['env'], d['cold_ms'], d['warm_ms'], d['x_ideal_cold'], d['win'], d['ef'], d['y_sha'])
PY
