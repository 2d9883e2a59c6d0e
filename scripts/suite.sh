#!/bin/bash
# dev (under gpurun): characterise BASELINE configs on one B200.
# usage: bash scripts/suite.sh TAG "1:original,random,rabbit,rabbitpp 3:original,rabbit,rabbitpp"
# Per config: one bench line (cold L2, all orderings) + an ncu pass over the exec
# kernels of each ordering (time, DRAM bytes, L2 hit) -> gpurun_out/suite_TAG_c*.
TAG=$1; SPECS=$2
mkdir -p gpurun_out /tmp/permcache
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv,noheader
lscpu | grep -E "^CPU\(s\)|Model name" ; free -g | head -2
for spec in $SPECS; do
  cfg=${spec%%:*}; ords=${spec#*:}
  echo "== config $cfg orderings $ords $(date +%T)"
  timeout ${BENCH_TO:-2400} python bench.py --config $cfg --orderings $ords --steps ${STEPS:-20} --warmup 3 \
      --no-cpu-baseline --perm-cache /tmp/permcache > gpurun_out/suite_${TAG}_c$cfg.json 2> gpurun_out/suite_${TAG}_c$cfg.err
  tail -2 gpurun_out/suite_${TAG}_c$cfg.err
  python - <<PY
import json; d=json.loads(open('gpurun_out/suite_${TAG}_c$cfg.json').read())
print(d['config']['workload'], d['config']['n'], d['config']['nnz'], 'ideal', d['config']['ideal_bytes'])
for k,v in d['orderings'].items(): print(' ', k, 'ms', v['ms'], 'warm', v['warm_ms'], 'x ideal', round(v['runtime_over_ideal'],3), 'reorder_s', round(v['reorder_s'],1), 'ins', round(v['insularity'],3), 'H', v['H'], 'win', v['l2_window_bytes'], 'ef', v['stream_evict_first'])
PY
  if [ -z "$SKIP_NCU" ]; then
  for ORD in ${ords//,/ }; do
    echo "-- ncu c$cfg $ORD $(date +%T)"
    timeout ${NCU_TO:-1200} ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct,l1tex__t_sector_hit_rate.pct \
      --clock-control none -k regex:"k_lane|k_warp_rows|k_cta_rows|k_hub|k_panel" -c 40 --csv \
      --log-file gpurun_out/suite_${TAG}_c${cfg}_${ORD}_ncu.csv \
      python bench.py --config $cfg --orderings $ORD --steps 2 --warmup 3 --no-cpu-baseline \
      --perm-cache /tmp/permcache > /dev/null 2>&1
  done
  fi
done
echo "end $(date +%T)"
