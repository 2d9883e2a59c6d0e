mkdir -p gpurun_out /tmp/permcache
STEPS=20 bash scripts/suite.sh r38 "2:rabbit,insular,hubgroup,hubsort,rabbitpp 3:rabbit,insular,hubgroup,hubsort,rabbitpp"
