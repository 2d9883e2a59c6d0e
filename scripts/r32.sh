mkdir -p gpurun_out /tmp/permcache
timeout 600 python -m pytest tests/test_gpu_spmm.py -x -q > gpurun_out/r32_tests.log 2>&1; tail -2 gpurun_out/r32_tests.log
timeout 300 python bench.py --steps 20 --no-cpu-baseline --orderings rabbitpp --perm-cache /tmp/permcache > gpurun_out/r32_bench.json 2> gpurun_out/r32_bench.err; tail -2 gpurun_out/r32_bench.err
python -c "
import json;d=json.loads(open('gpurun_out/r32_bench.json').read())
for k,v in d['orderings'].items(): print(k, v['ms'], v['runtime_over_ideal'], 'spmm4', v['spmm4'], 'coo', v['coo'])"
for K in k_lane4 "k_coo<"; do
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"$K" -s 2 -c 1 -o "gpurun_out/prof_r32_${K//</}" python bench.py --steps 3 --warmup 3 --orderings rabbitpp --no-cpu-baseline --perm-cache /tmp/permcache > /dev/null 2>&1
done
ls gpurun_out | grep r32
