# compute-sanitizer passes over the small GPU parity cases (under gpurun):
# memcheck (out-of-bounds / misaligned accesses, including the 256-bit
# chunk-rounded loads of k_lane / k_lane4 / k_coo_w that rely on the 8-element
# tail padding), racecheck and synccheck (shared-memory sorts, CTA-row
# reductions, the COO owner chain, k_panel's mbarrier ring, the register /
# shared-memory bitonic sorts and merge-path tiles of P A P^T, k_small's
# staged wide rows, the norm from y).  TO (seconds per tool) defaults to 2400.
mkdir -p gpurun_out
SEL="exec_matches_oracle or permute_and_bins or partitioned or smem_window or degenerate or iterate_regular or nonfinite or spmm or coo or every_sort_path or norm_from_y or lane_gather_policy"
for tool in memcheck racecheck synccheck; do
  timeout ${TO:-2400} compute-sanitizer --tool $tool --error-exitcode 99 --print-limit 20 \
    python -m pytest -q -x -m gpu tests/test_gpu_parity.py tests/test_gpu_nonfinite.py \
    tests/test_gpu_spmm.py tests/test_gpu_coo.py tests/test_gpu_permute_classes.py \
    tests/test_gpu_norm.py tests/test_gpu_lane_pred.py -k "$SEL and not full_size" \
    > gpurun_out/sanitize_$tool.log 2>&1
  echo "$tool rc=$?"; grep -E "ERROR SUMMARY|passed|failed" gpurun_out/sanitize_$tool.log | tail -3
done
