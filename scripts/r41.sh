mkdir -p gpurun_out /tmp/permcache
for CFG in 2 3; do
KIND=spmm4 CFG=$CFG ORDS=rabbitpp K=10 COMBOS='[{}, {"SPMV_L4_V": "1"}, {"SPMV_L4_V": "2"}]' timeout 1200 python scripts/knobs.py 2>&1 | grep -v Warn
done
