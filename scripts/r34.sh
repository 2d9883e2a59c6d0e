mkdir -p gpurun_out /tmp/permcache
BENCH_TO=3000 NCU_TO=1500 STEPS=10 bash scripts/suite.sh r34 "4:random,planted,rabbit,rabbitpp"
BENCH_TO=3000 NCU_TO=1500 STEPS=10 bash scripts/suite.sh r34 "5:original"
