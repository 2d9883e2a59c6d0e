#!/bin/bash
# dev (under gpurun): C3 RMAT-26 RABBIT++ launch list + ncu of the top kernels
mkdir -p gpurun_out /tmp/permcache
python bench.py --config 3 --orderings rabbitpp --steps 5 --warmup 3 --no-cpu-baseline --perm-cache /tmp/permcache > gpurun_out/c3_bench.json 2> gpurun_out/c3_bench.err
tail -c 600 gpurun_out/c3_bench.json
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,lts__t_sector_hit_rate.pct --clock-control none -c 200 --csv --log-file gpurun_out/c3_launches.csv python bench.py --config 3 --orderings rabbitpp --steps 2 --warmup 3 --no-cpu-baseline --perm-cache /tmp/permcache > /dev/null 2>&1
for K in k_lane k_warp_rows k_cta_rows k_hub_chunk; do
timeout 900 ncu --set full --clock-control none --import-source on -k regex:$K -s 3 -c 1 -o gpurun_out/prof_c3_$K python bench.py --config 3 --orderings rabbitpp --steps 2 --warmup 3 --no-cpu-baseline --perm-cache /tmp/permcache > /dev/null 2>&1
done
ls -la gpurun_out | grep c3
