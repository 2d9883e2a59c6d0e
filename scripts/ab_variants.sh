#!/bin/bash
# dev: A/B the short-row kernel variants on the bench workload (no ncu)
mkdir -p gpurun_out
TAG=${1:-ab}; shift
for V in 0 1; do
python bench.py --perm-cache /tmp/permcache --no-cpu-baseline --variant $V "$@" > gpurun_out/ab_${TAG}_v$V.json 2> gpurun_out/ab_${TAG}_v$V.err
python -c "
import json,sys; d=json.loads(open('gpurun_out/ab_${TAG}_v$V.json').read())
print('variant $V', {k:(round(v['ms'],4), round(v['runtime_over_ideal'],3)) for k,v in d['orderings'].items()})"
done
