mkdir -p gpurun_out /tmp/permcache
timeout 1200 python -m pytest tests/test_gpu_spmm.py tests/test_gpu_parity.py tests/test_gpu_fused.py -x -q > gpurun_out/r42_tests.log 2>&1; tail -3 gpurun_out/r42_tests.log
KIND=exec CFG=3 ORDS=rabbitpp,hubsort K=10 COMBOS='[{}]' timeout 1200 python scripts/knobs.py 2>&1 | grep -v Warn
KIND=exec CFG=2 ORDS=rabbitpp K=20 COMBOS='[{}]' timeout 600 python scripts/knobs.py 2>&1 | grep -v Warn
