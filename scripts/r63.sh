# round 2: both factors masked in k_lane vs the round-1 schedule (C2), same box
for c in 4375ce7 mask2 4375ce7 mask2; do
  timeout 600 python scratch_old/c2time.py scratch_old/$c 2>> gpurun_out/r63.err | tail -1
done
