# round 2: C2 exec vs round 1 after the value-mask split; targeted GPU tests; compute-sanitizer
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r64_build.log 2>&1 || tail -20 gpurun_out/r64_build.log
for c in 4375ce7 mask3; do timeout 600 python scratch_old/c2time.py scratch_old/$c 2>> gpurun_out/r64.err | tail -1; done
timeout 1200 python -m pytest -q -m gpu tests/test_gpu_nonfinite.py tests/test_gpu_spmm.py tests/test_gpu_unroll.py "tests/test_gpu_parity.py::test_exec_matches_oracle" "tests/test_gpu_parity.py::test_small_plan_single_launch_bitwise" > gpurun_out/r64_tests.log 2>&1; echo "tests rc=$?"; tail -3 gpurun_out/r64_tests.log
bash scripts/sanitize.sh
