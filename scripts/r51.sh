# C1 (RMAT-16, L2-resident, launch bound): fork/join and grid knobs
mkdir -p gpurun_out
C='[{}, {"SPMV_CONCURRENT": "0"}, {"SPMV_FORK_EARLY": "0"}, {"SPMV_LANE_CTAS": "1"}, {"SPMV_LANE_CTAS": "2"}, {"SPMV_WIN_COLS": "0"}, {}]'
KIND=exec CFG=1 ORDS=original,rabbit,rabbitpp K=50 COMBOS="$C" timeout 600 python scripts/knobs.py 2>&1 | grep -v Warn | tee gpurun_out/r51_c1_knobs.log
