# round 2, first box call: new parity tests + host specs + generator timings
mkdir -p gpurun_out
nproc > gpurun_out/r52_host.txt; lscpu >> gpurun_out/r52_host.txt; free -g >> gpurun_out/r52_host.txt; nvidia-smi -L >> gpurun_out/r52_host.txt
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r52_build.log 2>&1
timeout 900 python -m pytest -q -m gpu tests/test_gpu_nonfinite.py tests/test_gpu_iterate_dist.py tests/test_gpu_fused.py "tests/test_gpu_parity.py::test_partitioned_equals_single_bitwise" "tests/test_gpu_parity.py::test_iterate_matches_oracle_recurrence" "tests/test_gpu_parity.py::test_errors" > gpurun_out/r52_tests.log 2>&1; tail -30 gpurun_out/r52_tests.log
timeout 1500 python - > gpurun_out/r52_gen.log 2>&1 <<'PY'
import time, sys
sys.path.insert(0, '.')
import synth
for k in (3, 4, 5):
    t = time.time(); w = synth.config(k); print(k, w.name, w.A.n, w.A.nnz, 'gen_s', round(time.time() - t, 1), flush=True)
    del w
PY
cat gpurun_out/r52_gen.log
