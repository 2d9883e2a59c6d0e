mkdir -p gpurun_out /tmp/permcache
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r79_build.log 2>&1 || tail -20 gpurun_out/r79_build.log
timeout 1500 python -m pytest -q -m gpu tests/test_gpu_permute_classes.py "tests/test_gpu_parity.py::test_permute_and_bins_bitexact" tests/test_gpu_lane_pred.py "tests/test_gpu_parity.py::test_exec_matches_oracle" > gpurun_out/r79_tests.log 2>&1; echo "tests rc=$?"; tail -2 gpurun_out/r79_tests.log
for co in "5 rabbitpp" "3 rabbitpp" "1 rabbitpp" "2 rabbitpp"; do set -- $co
  it=""; [ "$1" = 5 ] && it="--iterate"
  for rep in 1 2; do
    for e in SPMV_LANE_ONE=0 SPMV_LANE_ONE=1; do
      timeout 1200 python scripts/kprof.py --config $1 --ordering $2 --steps 10 $it --env $e >> gpurun_out/r79_ab.jsonl 2>> gpurun_out/r79_ab.err
    done
  done
done
python - <<'PY'
import json
for l in open('gpurun_out/r79_ab.jsonl'):
    d=json.loads(l); print(d['workload'], d['env'], 'cold', d['cold_ms'], 'warm', d['warm_ms'], 'scaled', d['scaled_fixed_ms'], 'it', d['iterate_ms'], d['y_sha'], 'permute', d.get('permute_ms'), 'lane_nnz', d.get('lane_nnz'))
PY
for e in SPMV_LANE_ONE=0 SPMV_LANE_ONE=1; do
  timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,launch__registers_per_thread --cache-control none --clock-control none -k regex:"k_lane" --csv --log-file gpurun_out/r79_c5_$e.csv python scripts/kprof.py --config 5 --ordering rabbitpp --ncu 2 --env $e > /dev/null 2>&1
  python scripts/ncu_list.py gpurun_out/r79_c5_$e.csv | tail -2 | cut -c1-150
done
