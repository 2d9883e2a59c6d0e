mkdir -p gpurun_out /tmp/permcache
timeout 1500 python -m pytest tests -x -q -m gpu > gpurun_out/r39_tests.log 2>&1; tail -3 gpurun_out/r39_tests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r39_smoke.log 2>&1; tail -2 gpurun_out/r39_smoke.log
SKIP_TESTS=1 bash scripts/gpu_bench_profile.sh r39
timeout 1800 python bench.py --config 3 --orderings rabbitpp --steps 10 --no-cpu-baseline --perm-cache /tmp/permcache > gpurun_out/r39_c3.json 2> gpurun_out/r39_c3.err
python -c "
import json;d=json.loads(open('gpurun_out/r39_c3.json').read())
for k,v in d['orderings'].items(): print('c3', k, v['ms'], v['runtime_over_ideal'], 'reorder', v['reorder_s'], 'spmm4', v['spmm4'], 'coo', v['coo'])"
