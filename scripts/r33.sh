mkdir -p gpurun_out /tmp/permcache
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "hot or exec_matches or partitioned or graph or iterate" > gpurun_out/r33_tests.log 2>&1; tail -3 gpurun_out/r33_tests.log
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"k_coo[^_]" -s 2 -c 1 -o gpurun_out/prof_r33_k_coo python bench.py --steps 3 --warmup 3 --orderings rabbitpp --no-cpu-baseline > gpurun_out/r33_ncu_coo.log 2>&1
CFG=3 ORDS=rabbitpp COMBOS='[{"SPMV_HOT": "-1"}, {}, {"SPMV_HOT_COLD": "0"}, {"SPMV_FORK_EARLY": "0"}, {"SPMV_HOT": "-1", "SPMV_FORK_EARLY": "0"}, {"SPMV_CONCURRENT": "0"}]' timeout 1500 python scripts/knobs.py > gpurun_out/r33_knobs.log 2>&1; cat gpurun_out/r33_knobs.log | tail -7
for H in -1 0; do
SPMV_HOT=$H timeout 900 ncu --set full --clock-control none -k regex:k_warp_rows -s 2 -c 1 -o gpurun_out/prof_r33_c3_warp_hot$H python bench.py --config 3 --orderings rabbitpp --steps 2 --warmup 3 --no-cpu-baseline --no-side --perm-cache /tmp/permcache > /dev/null 2>&1
done
ls gpurun_out | grep r33
