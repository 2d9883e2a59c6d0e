# round 2 (session 2): iterate window alternation A/B (half vs full window), interleaved processes;
# C1-C5 suite (cold SpMV per config, C5 iterate) -> geomean of runtime / ideal
mkdir -p gpurun_out /tmp/permcache
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r74_build.log 2>&1 || tail -20 gpurun_out/r74_build.log
timeout 1200 python -m pytest -q -m gpu "tests/test_gpu_parity.py::test_small_plan_single_launch_bitwise" tests/test_gpu_lane_pred.py > gpurun_out/r74_tests.log 2>&1; echo "tests rc=$?"; tail -2 gpurun_out/r74_tests.log
for so in variants/head.so paper_conf_ispass_balajicjk23_b200/libspmv.so variants/head.so paper_conf_ispass_balajicjk23_b200/libspmv.so; do
  timeout 600 python scripts/kprof.py --config 1 --ordering rabbitpp --steps 30 --so $so 2>> gpurun_out/r74_c1.err | python -c "import sys,json; d=json.loads(sys.stdin.read()); print('C1', d['so'], d['cold_ms'], d['warm_ms'], d['y_sha'])"
done
for rep in 1 2; do
  for e in SPMV_WIN_ALT_FULL=0 SPMV_WIN_ALT_FULL=1; do
    timeout 1200 python scripts/kprof.py --config 5 --ordering rabbitpp --steps 10 --iterate --env $e >> gpurun_out/r74_alt.jsonl 2>> gpurun_out/r74_alt.err
  done
done
python - <<'PY'
import json
for l in open('gpurun_out/r74_alt.jsonl'):
    d=json.loads(l); print(d['env'], 'cold', d['cold_ms'], 'warm', d['warm_ms'], 'scaled', d['scaled_fixed_ms'], 'it', d['iterate_ms'], 'win', d['win'])
PY
timeout 3600 python scripts/suite.py --out gpurun_out/suite_r74.json > gpurun_out/r74_suite.log 2>&1; echo "suite rc=$?"; tail -3 gpurun_out/r74_suite.log
