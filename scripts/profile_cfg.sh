#!/bin/bash
# dev (under gpurun): ncu --set full of one exec kernel on config CFG, ordering ORD
# usage: CFG=4 ORD=planted K=k_lane bash scripts/profile_cfg.sh
mkdir -p gpurun_out /tmp/permcache
CFG=${CFG:-4}; ORD=${ORD:-planted}; K=${K:-k_lane}
timeout 1500 ncu --set full --clock-control none --import-source on -k regex:$K -s ${SKIP:-2} -c 1 \
  -o gpurun_out/prof_c${CFG}_${ORD}_$K python bench.py --config $CFG --orderings $ORD --steps 2 --warmup 3 \
  --no-cpu-baseline --perm-cache /tmp/permcache > gpurun_out/prof_c${CFG}_${ORD}_$K.log 2>&1
tail -3 gpurun_out/prof_c${CFG}_${ORD}_$K.log
