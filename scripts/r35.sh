mkdir -p gpurun_out /tmp/permcache
timeout 900 python -m pytest tests/test_gpu_coo.py tests/test_gpu_spmm.py tests/test_gpu_parity.py -x -q -k "coo or spmm or hot or graph or exec_matches" > gpurun_out/r35_tests.log 2>&1; tail -3 gpurun_out/r35_tests.log
for V in 2 1; do
SPMV_COO_V=$V timeout 300 python bench.py --steps 20 --no-cpu-baseline --orderings rabbitpp --perm-cache /tmp/permcache > gpurun_out/r35_bench_coo$V.json 2> gpurun_out/r35_bench_coo$V.err
python -c "
import json;d=json.loads(open('gpurun_out/r35_bench_coo$V.json').read())
for k,v in d['orderings'].items(): print('coo v$V', k, v['ms'], v['runtime_over_ideal'], 'graph', v['graph_warm_ms'], 'spmm4', v['spmm4']['ms'], v['spmm4']['runtime_over_ideal'], 'coo', v['coo']['ms'], v['coo']['runtime_over_ideal'])"
done
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"k_coo_w" -s 2 -c 1 -o gpurun_out/prof_r35_k_coo_w python bench.py --steps 3 --warmup 3 --orderings rabbitpp --no-cpu-baseline --perm-cache /tmp/permcache > /dev/null 2>&1
CFG=3 ORDS=rabbitpp COMBOS='[{"SPMV_HOT": "-1"}, {"SPMV_HOT": "1"}, {"SPMV_HOT": "1", "SPMV_HOT_MODE": "1"}, {"SPMV_HOT": "1", "SPMV_FORK_EARLY": "0"}]' timeout 1500 python scripts/knobs.py > gpurun_out/r35_knobs.log 2>&1; cat gpurun_out/r35_knobs.log | tail -5
SPMV_HOT=1 timeout 900 ncu --set full --clock-control none -k regex:"k_warp_rows_smem|k_long_rows_smem" -s 2 -c 2 -o gpurun_out/prof_r35_c3_smem python bench.py --config 3 --orderings rabbitpp --steps 2 --warmup 3 --no-cpu-baseline --no-side --perm-cache /tmp/permcache > /dev/null 2>&1
ls gpurun_out | grep r35
