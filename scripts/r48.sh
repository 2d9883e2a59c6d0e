# k_warp_rows entries in flight per lane: 4 (default) vs 8 (SPMV_WARP_UNR=8), same association
mkdir -p gpurun_out /tmp/permcache
SPMV_WARP_UNR=8 timeout 900 python -m pytest tests/test_gpu_parity.py -x -q > gpurun_out/r48_tests.log 2>&1; tail -3 gpurun_out/r48_tests.log
C='[{}, {"SPMV_WARP_UNR": "8"}, {}]'
KIND=exec CFG=1 ORDS=original,rabbitpp K=30 COMBOS="$C" timeout 300 python scripts/knobs.py 2>&1 | grep -v Warn
KIND=exec CFG=2 ORDS=rabbitpp K=20 COMBOS="$C" timeout 600 python scripts/knobs.py 2>&1 | grep -v Warn
KIND=exec CFG=3 ORDS=rabbitpp,original K=10 COMBOS="$C" timeout 1500 python scripts/knobs.py 2>&1 | grep -v Warn
