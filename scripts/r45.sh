mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_bench_multirank.py tests/test_gpu_parity.py -x -q -k "two_ranks or stencil464" > gpurun_out/r45_tests.log 2>&1; tail -3 gpurun_out/r45_tests.log
timeout 400 python bench.py > gpurun_out/r45_bench.json 2> gpurun_out/r45_bench.err; tail -2 gpurun_out/r45_bench.err
python -c "
import json;d=json.loads(open('gpurun_out/r45_bench.json').read())
print(d['value'], d['ms_per_step'], d['runtime_over_ideal'], d['e2e'], d['gpu_launches'], d['cpu_baseline']['value'])"
