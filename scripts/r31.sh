mkdir -p gpurun_out
python scripts/devattr.py > gpurun_out/r31_devattr.txt 2>&1; cat gpurun_out/r31_devattr.txt
timeout 900 python -m pytest tests/test_gpu_spmm.py tests/test_gpu_coo.py -x -q > gpurun_out/r31_tests.log 2>&1; tail -15 gpurun_out/r31_tests.log
timeout 300 python bench.py --steps 20 --no-cpu-baseline --orderings original,rabbitpp > gpurun_out/r31_bench.json 2> gpurun_out/r31_bench.err; tail -3 gpurun_out/r31_bench.err
CFG=3 ORDS=rabbitpp COMBOS='[{}, {"SPMV_L2_FETCH": "32"}, {"SPMV_L2_FETCH": "128"}, {"SPMV_WIN_COLS": "8000000"}, {"SPMV_WIN_COLS": "16000000"}, {"SPMV_WIN_COLS": "24000000"}, {"SPMV_WIN_ALL": "1"}, {"SPMV_LANE_EF": "1"}, {"SPMV_CONCURRENT": "0"}, {"SPMV_LANE_GL": "1"}]' timeout 1500 python scripts/knobs.py > gpurun_out/r31_knobs.log 2>&1; cat gpurun_out/r31_knobs.log | tail -14
