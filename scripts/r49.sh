# warp / CTA row kernels: 4 vs 8 entries in flight (SPMV_WARP_UNR, SPMV_CTA_UNR), same association
mkdir -p gpurun_out /tmp/permcache
timeout 900 python -m pytest tests/test_gpu_unroll.py -x -q > gpurun_out/r49_tests.log 2>&1; tail -2 gpurun_out/r49_tests.log
SPMV_WARP_UNR=8 SPMV_CTA_UNR=8 timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fused.py -x -q >> gpurun_out/r49_tests.log 2>&1; tail -2 gpurun_out/r49_tests.log
C='[{}, {"SPMV_WARP_UNR": "8"}, {"SPMV_CTA_UNR": "8"}, {"SPMV_WARP_UNR": "8", "SPMV_CTA_UNR": "8"}, {}]'
KIND=exec CFG=1 ORDS=original,rabbitpp K=30 COMBOS="$C" timeout 300 python scripts/knobs.py 2>&1 | grep -v Warn
KIND=exec CFG=2 ORDS=rabbitpp K=20 COMBOS="$C" timeout 600 python scripts/knobs.py 2>&1 | grep -v Warn
KIND=exec CFG=3 ORDS=rabbitpp K=10 COMBOS="$C" timeout 1500 python scripts/knobs.py 2>&1 | grep -v Warn
