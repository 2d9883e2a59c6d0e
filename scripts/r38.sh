mkdir -p gpurun_out /tmp/permcache
timeout 900 python -m pytest tests/test_gpu_fused.py tests/test_gpu_bench_multirank.py tests/test_gpu_parity.py -x -q -k "fused or bcast or partitioned or iterate or hot or two_ranks" > gpurun_out/r38_tests.log 2>&1; tail -15 gpurun_out/r38_tests.log
SPMV_COO_MINB=4 timeout 300 python bench.py --steps 20 --no-cpu-baseline --orderings rabbitpp --perm-cache /tmp/permcache > gpurun_out/r38_coo_minb4.json 2>/dev/null
python -c "
import json;d=json.loads(open('gpurun_out/r38_coo_minb4.json').read())
for k,v in d['orderings'].items(): print('minb4', k, 'coo', v['coo'])"
STEPS=20 bash scripts/suite.sh r38 "2:rabbit,insular,hubgroup,hubsort,rabbitpp 3:rabbit,insular,hubgroup,hubsort,rabbitpp"
