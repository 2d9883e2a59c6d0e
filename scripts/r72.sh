# round 2 (session 2): where exec_scaled's extra time goes (norm partial stores) and the
# predicated k_lane at 64 registers (4 CTAs/SM)
mkdir -p gpurun_out /tmp/permcache
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r72_build.log 2>&1 || tail -20 gpurun_out/r72_build.log
timeout 1200 python -m pytest -q -m gpu "tests/test_gpu_parity.py::test_small_plan_single_launch_bitwise" tests/test_gpu_permute_classes.py > gpurun_out/r72_tests.log 2>&1; echo "tests rc=$?"; tail -3 gpurun_out/r72_tests.log
for so in variants/head.so paper_conf_ispass_balajicjk23_b200/libspmv.so; do
  timeout 600 python scripts/kprof.py --config 1 --ordering rabbitpp --steps 20 --so $so >> gpurun_out/r72_ab.jsonl 2>> gpurun_out/r72_ab.err
done
for so in paper_conf_ispass_balajicjk23_b200/libspmv.so variants/noss.so; do
  timeout 1200 python scripts/kprof.py --config 5 --ordering rabbitpp --steps 10 --iterate --so $so >> gpurun_out/r72_ab.jsonl 2>> gpurun_out/r72_ab.err
done
for co in "4 rabbit" "4 rabbitpp" "2 rabbitpp"; do set -- $co
  for so in paper_conf_ispass_balajicjk23_b200/libspmv.so variants/predm4.so; do
    timeout 1200 python scripts/kprof.py --config $1 --ordering $2 --steps 10 --env SPMV_LANE_PRED=1 --so $so >> gpurun_out/r72_ab.jsonl 2>> gpurun_out/r72_ab.err
  done
done
python - <<'PY'
import json
for l in open('gpurun_out/r72_ab.jsonl'):
    d=json.loads(l); print(d['workload'], d['ordering'], (d['so'] or '').split('/')[-1], d['env'], 'cold', d['cold_ms'], 'warm', d['warm_ms'], 'scaled', d['scaled_fixed_ms'], 'it', d['iterate_ms'], d['y_sha'], d.get('permute_ms'))
PY
