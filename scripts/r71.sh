# round 2 (session 2): P A P^T rework (register sort of rows 33..256, tiled big-row chunk sort,
# merge-path passes): bit-exact tests, permute time on C1-C5, launch list of the C5 permute
mkdir -p gpurun_out /tmp/permcache
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r71_build.log 2>&1 || tail -20 gpurun_out/r71_build.log
timeout 1500 python -m pytest -q -m gpu tests/test_gpu_permute_classes.py "tests/test_gpu_parity.py::test_permute_and_bins_bitexact" tests/test_gpu_parity.py::test_rmat16_full_size tests/test_gpu_parity.py::test_iterate_matches_oracle_recurrence tests/test_gpu_parity.py::test_rmat26_rabbitpp_full_size > gpurun_out/r71_tests.log 2>&1; echo "tests rc=$?"; tail -3 gpurun_out/r71_tests.log
for co in "1 rabbitpp" "2 rabbitpp" "3 rabbitpp" "4 rabbitpp" "5 rabbitpp"; do set -- $co
  for so in variants/head.so paper_conf_ispass_balajicjk23_b200/libspmv.so; do
    timeout 1200 python scripts/kprof.py --config $1 --ordering $2 --steps 5 --so $so >> gpurun_out/r71_kprof.jsonl 2>> gpurun_out/r71_kprof.err
  done
done
python - <<'PY'
import json
for l in open('gpurun_out/r71_kprof.jsonl'):
    d=json.loads(l); print(d['workload'], (d['so'] or 'tree').split('/')[-1], 'plan_s', d.get('plan_s'), 'permute_ms', d.get('permute_ms'), 'cold', d['cold_ms'], d['y_sha'])
PY
timeout 1200 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/r71_c5_permute.csv python scripts/kprof.py --config 5 --ordering rabbitpp --ncu 1 > gpurun_out/r71_ncu.log 2>&1; echo "ncu rc=$?"
