#!/bin/bash
# Characterise other BASELINE configs (dev, under gpurun): one bench line per config.
# usage: bash scripts/characterize.sh "1:original,random,rabbit,rabbitpp 3:original,rabbit,rabbitpp"
mkdir -p gpurun_out /tmp/permcache
for spec in $1; do
  cfg=${spec%%:*}; ords=${spec#*:}
  echo "== config $cfg orderings $ords"; date
  timeout 3000 python bench.py --config $cfg --orderings $ords --steps ${STEPS:-20} --warmup 3 \
      --no-cpu-baseline --perm-cache /tmp/permcache > gpurun_out/char_c$cfg.json 2> gpurun_out/char_c$cfg.err
  tail -3 gpurun_out/char_c$cfg.err
  python -c "
import json; d=json.loads(open('gpurun_out/char_c$cfg.json').read())
print(d['config']['workload'], d['config']['n'], d['config']['nnz'])
for k,v in d['orderings'].items(): print(' ', k, 'ms', v['ms'], 'warm', v['warm_ms'], 'x ideal', round(v['runtime_over_ideal'],3), 'reorder_s', round(v['reorder_s'],1), 'ins', round(v['insularity'],3), 'skew', round(v['skew'],3))
"
done
