# round 2: full GPU suite + smoke, then C5 studies (iterate overhead fixed, HUBSORT), Fig. 6, C3 reorder
mkdir -p gpurun_out /tmp/permcache
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r55_build.log 2>&1 || tail -20 gpurun_out/r55_build.log
timeout 2400 python -m pytest tests -q -m gpu -x > gpurun_out/r55_tests.log 2>&1; echo "tests rc=$?"; tail -15 gpurun_out/r55_tests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -2
for o in rabbitpp hubsort; do
  SPMV_REORDER_VERBOSE=1 timeout 900 python scripts/kprof.py --config 5 --ordering $o --steps 10 --iterate >> gpurun_out/r55_kprof.log 2>> gpurun_out/r55_kprof.err; echo "kprof $o rc=$?"
done
cat gpurun_out/r55_kprof.log; grep "par:\|deferred\|stats\|symm\|detect" gpurun_out/r55_kprof.err | tail -10
for c in 2 3; do timeout 900 python scripts/fig6.py --config $c >> gpurun_out/r55_fig6.log 2>&1; done; cat gpurun_out/r55_fig6.log
