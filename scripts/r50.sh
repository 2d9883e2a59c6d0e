mkdir -p gpurun_out
timeout 1800 python -m pytest tests -q -m gpu > gpurun_out/r50_tests.log 2>&1; tail -3 gpurun_out/r50_tests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
timeout 400 python bench.py > gpurun_out/r50_bench.json 2> gpurun_out/r50_bench.err; tail -2 gpurun_out/r50_bench.err
python -c "
import json;d=json.loads(open('gpurun_out/r50_bench.json').read())
print(d['value'], d['ms_per_step'], d['runtime_over_ideal'], d['roofline']['frac'], d['e2e']['ms_per_step'], d['gpu_launches'], d['clocks'])"
timeout 600 python bench.py --impl reference --steps 5 --warmup 3 > gpurun_out/r50_ref.json 2>/dev/null; cut -c1-300 gpurun_out/r50_ref.json
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/r50_launches.csv python bench.py --steps 2 --warmup 3 > gpurun_out/r50_ncu_bench.log 2>&1; wc -l gpurun_out/r50_launches.csv
