mkdir -p gpurun_out /tmp/permcache
nproc; free -g | head -2
BENCH_TO=3300 SKIP_NCU=1 STEPS=10 bash scripts/suite.sh r37 "5:rabbitpp"
