#!/bin/bash
# DRAM traffic of every k_advance launch of one profiled run (the same launches bench.py's roofline
# averages over): writes gpurun_out/traffic_<config>_<alg>.csv
cfg=$1; alg=$2
timeout 900 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none \
  -k regex:k_advance --csv --log-file gpurun_out/traffic_${cfg}_${alg}.csv \
  python tools/profile_run.py --config $cfg --alg $alg --runs 1 > gpurun_out/traffic_${cfg}_${alg}.log 2>&1
echo "traffic $cfg $alg rc=$?"
