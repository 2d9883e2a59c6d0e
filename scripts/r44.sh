mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "rabbitpp_gpu" > gpurun_out/r44_tests.log 2>&1; tail -2 gpurun_out/r44_tests.log
timeout 1200 python scripts/postpass_c3.py 3 2>&1 | tail -1 | tee gpurun_out/r44_postpass_c3.json
timeout 300 python bench.py --config 1 --orderings original,rabbitpp --steps 50 --no-cpu-baseline > gpurun_out/r44_c1.json 2>/dev/null
python -c "
import json;d=json.loads(open('gpurun_out/r44_c1.json').read())
for k,v in d['orderings'].items(): print('c1', k, 'cold', v['ms'], 'warm', v['warm_ms'], 'graph', v['graph_warm_ms'], 'spmm4', v['spmm4']['ms'], 'coo', v['coo']['ms'])"
