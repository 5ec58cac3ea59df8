#!/bin/bash
# Round measurements (1 GPU) -- bench lines for every config, ablations, ncu evidence for the advance.
mkdir -p gpurun_out/m2
timeout 600 python bench.py > gpurun_out/m2/bench_C2.json 2> gpurun_out/m2/bench_C2.err; echo "C2 rc=$?"
timeout 300 python bench.py --config C1 --steps 50 > gpurun_out/m2/bench_C1.json 2> gpurun_out/m2/bench_C1.err; echo "C1 rc=$?"
timeout 900 python bench.py --config C3 --steps 3 --warmup 3 --no-e2e > gpurun_out/m2/bench_C3.json 2> gpurun_out/m2/bench_C3.err; echo "C3 rc=$?"
timeout 900 python bench.py --config C4 --steps 5 --warmup 3 --no-e2e > gpurun_out/m2/bench_C4.json 2> gpurun_out/m2/bench_C4.err; echo "C4 rc=$?"
timeout 900 python bench.py --config C5 --steps 3 --warmup 3 --no-e2e > gpurun_out/m2/bench_C5.json 2> gpurun_out/m2/bench_C5.err; echo "C5 rc=$?"
timeout 900 python bench.py --impl reference --steps 3 > gpurun_out/m2/bench_ref_C2.json 2> gpurun_out/m2/bench_ref_C2.err; echo "ref rc=$?"
for cfg in "C2 bfs 3" "C5 pr 2" "C4 wcc 1"; do set -- $cfg
  timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/m2/launches_$1_$2.csv python tools/profile_run.py --config $1 --alg $2 --runs 1 > /dev/null 2>&1
  timeout 900 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none -k regex:k_advance --csv --log-file gpurun_out/m2/traffic_$1_$2.csv python tools/profile_run.py --config $1 --alg $2 --runs 1 > /dev/null 2>&1
  timeout 900 ncu --set full --import-source on --clock-control none -k regex:k_advance -s $3 -c 1 -o gpurun_out/m2/adv_$1_$2 python tools/profile_run.py --config $1 --alg $2 --runs 1 > /dev/null 2>&1
  echo "ncu $1 $2 rc=$?"
done
