# round 2: A/B of the next-row prefetch in k_warp_rows (pre = HEAD, post = working tree), C3 and C5
mkdir -p gpurun_out /tmp/permcache
for t in pre post; do (cd scratch_old/$t && python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1); done
for rep in 1 2; do for t in pre post; do for c in 3 5; do
  (cd scratch_old/$t && timeout 900 python scripts/kprof.py --config $c --ordering rabbitpp --steps 10 --iterate 2>>../../gpurun_out/r65.err | python -c "import sys,json; d=json.loads(sys.stdin.read()); print('$t', d['workload'], d['cold_ms'], d['warm_ms'], d['iterate_ms'], d['y_sha'])")
done; done; done
