# round 2: GPU tests of the new code + first C5 bench (default) + reference arm
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r53_build.log 2>&1 || tail -20 gpurun_out/r53_build.log
timeout 900 python -m pytest -q -m gpu tests/test_synth_gpu.py tests/test_gpu_bench_multirank.py tests/test_gpu_iterate_dist.py > gpurun_out/r53_tests_new.log 2>&1; tail -5 gpurun_out/r53_tests_new.log
SPMV_REORDER_VERBOSE=1 timeout 1500 python bench.py --steps 20 --warmup 5 > gpurun_out/r53_bench.json 2> gpurun_out/r53_bench.err; echo "bench rc=$?"; tail -30 gpurun_out/r53_bench.err | grep -v "^$" | tail -25
python -c "
import json;d=json.loads(open('gpurun_out/r53_bench.json').read())
print(d['value'], d['ms_per_step'], d['runtime_over_ideal'], d['roofline']['frac'], d['e2e'], d['gpu_launches'], d['clocks'], d['input_prep'])
for k,v in d['orderings'].items(): print(k, v)
print(d.get('cpu_baseline'))"
timeout 900 python bench.py --impl reference --steps 5 --warmup 3 > gpurun_out/r53_ref.json 2> gpurun_out/r53_ref.err; echo "ref rc=$?"; cut -c1-600 gpurun_out/r53_ref.json; tail -3 gpurun_out/r53_ref.err
