# round 2: C1-C5 suite (geomean of runtime / ideal) -> profiles
mkdir -p gpurun_out /tmp/permcache
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r60_build.log 2>&1 || tail -20 gpurun_out/r60_build.log
SPMV_REORDER_VERBOSE=1 timeout 5000 python scripts/suite.py --configs 1,2,3,4,5 --steps 10 --out gpurun_out/suite_r60.json 2> gpurun_out/r60_suite.err | tee gpurun_out/r60_suite.log
