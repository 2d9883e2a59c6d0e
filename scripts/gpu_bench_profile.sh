#!/bin/bash
# dev helper (run under gpurun): GPU tests, bench, ncu launch list, ncu --set full of the stream kernel
# usage: bash scripts/gpu_bench_profile.sh TAG [extra bench args]
TAG=${1:-dev}; shift
mkdir -p gpurun_out
if [ -z "$SKIP_TESTS" ]; then timeout 900 python -m pytest tests -x -q -m gpu > gpurun_out/tests_$TAG.log 2>&1; tail -3 gpurun_out/tests_$TAG.log; fi
python bench.py --perm-cache /tmp/permcache "$@" > gpurun_out/bench_$TAG.json 2> gpurun_out/bench_$TAG.err
tail -c 1500 gpurun_out/bench_$TAG.json; tail -5 gpurun_out/bench_$TAG.err
if [ -z "$SKIP_NCU" ]; then
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches_$TAG.csv python bench.py --steps 5 --warmup 3 --orderings rabbitpp --no-cpu-baseline --perm-cache /tmp/permcache "$@" > /dev/null 2>&1
for ORD in ${NCU_ORDS:-rabbitpp original}; do
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_lane -s 3 -c 1 -o gpurun_out/prof_${TAG}_$ORD python bench.py --steps 3 --warmup 3 --orderings $ORD --no-cpu-baseline --perm-cache /tmp/permcache "$@" --orderings $ORD > gpurun_out/ncu_${TAG}_$ORD.log 2>&1
done
fi
ls gpurun_out
