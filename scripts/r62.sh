# round 2: which part of 6723b83 slowed C2 (use_device in spmv_exec? the product select?)
for c in 4375ce7 HEAD nodev oldmask both; do
  timeout 600 python scratch_old/c2time.py scratch_old/$c 2>> gpurun_out/r62.err | tail -1
done
