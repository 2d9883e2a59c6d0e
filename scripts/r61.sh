# round 2: bisect the C2 exec regression across the round-2 commits (same box)
for c in 4375ce7 6723b83 07f09a9 760a54e b6fb1a1 ae65fb5 589c8f9 b5feb5b HEAD; do
  timeout 600 python scratch_old/c2time.py scratch_old/$c 2>> gpurun_out/r61.err | tail -1
done
