#!/bin/bash
# All round measurements (1 GPU): bench lines for every config, ablations, launch lists, traffic.
mkdir -p gpurun_out/m
timeout 500 python bench.py > gpurun_out/m/bench_C2.json 2> gpurun_out/m/bench_C2.err; echo "C2 rc=$?"
timeout 300 python bench.py --config C1 --steps 50 > gpurun_out/m/bench_C1.json 2> gpurun_out/m/bench_C1.err; echo "C1 rc=$?"
timeout 900 python bench.py --config C3 --steps 3 --warmup 3 --no-e2e > gpurun_out/m/bench_C3.json 2> gpurun_out/m/bench_C3.err; echo "C3 rc=$?"
timeout 900 python bench.py --config C4 --steps 5 --warmup 3 --no-e2e > gpurun_out/m/bench_C4.json 2> gpurun_out/m/bench_C4.err; echo "C4 rc=$?"
timeout 900 python bench.py --config C5 --steps 3 --warmup 3 --no-e2e > gpurun_out/m/bench_C5.json 2> gpurun_out/m/bench_C5.err; echo "C5 rc=$?"
timeout 600 python tools/ablation.py --fsteal --scale 22 --workers 8 --out gpurun_out/m/abl_fsteal_virtual.json
timeout 600 python tools/ablation.py --fsteal --scale 22 --workers 8 --split --out gpurun_out/m/abl_fsteal_split.json
timeout 900 python tools/ablation.py --osteal --grid 2048 --workers 8 --delta 1024 --out gpurun_out/m/abl_osteal_virtual.json
timeout 900 python tools/c3_sweep.py 0,1024,4096 > gpurun_out/m/c3_sweep.jsonl 2>&1
for cfg in "C2 bfs" "C5 pr" "C4 wcc"; do set -- $cfg
  timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/m/launches_$1_$2.csv python tools/profile_run.py --config $1 --alg $2 --runs 1 > /dev/null 2>&1
  timeout 900 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none -k regex:k_advance --csv --log-file gpurun_out/m/traffic_$1_$2.csv python tools/profile_run.py --config $1 --alg $2 --runs 1 > /dev/null 2>&1
  echo "ncu $1 $2 rc=$?"
done
