#!/bin/bash
# Round measurements after the session-2 kernel work (1 GPU): bench lines for every config, the reference
# arm, launch lists, advance DRAM traffic, ncu --set full of the C2 peak advance and filter, ablations.
O=gpurun_out/m3; mkdir -p $O
timeout 500 python bench.py > $O/bench_C2.json 2> $O/bench_C2.err; echo "C2 rc=$?"
timeout 300 python bench.py --config C1 --steps 50 > $O/bench_C1.json 2> $O/bench_C1.err; echo "C1 rc=$?"
timeout 900 python bench.py --config C3 --steps 3 --warmup 3 --no-e2e > $O/bench_C3.json 2> $O/bench_C3.err; echo "C3 rc=$?"
timeout 900 python bench.py --config C4 --steps 5 --warmup 3 --no-e2e > $O/bench_C4.json 2> $O/bench_C4.err; echo "C4 rc=$?"
timeout 900 python bench.py --config C5 --steps 3 --warmup 3 --no-e2e > $O/bench_C5.json 2> $O/bench_C5.err; echo "C5 rc=$?"
timeout 600 python bench.py --impl reference --steps 3 > $O/bench_ref_C2.json 2> $O/bench_ref_C2.err; echo "ref rc=$?"
for cfg in "C2 bfs" "C5 pr" "C4 wcc"; do set -- $cfg
  timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_$1_$2.csv python tools/profile_run.py --config $1 --alg $2 --runs 1 > /dev/null 2>&1
  timeout 900 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none -k regex:k_advance --csv --log-file $O/traffic_$1_$2.csv python tools/profile_run.py --config $1 --alg $2 --runs 1 > /dev/null 2>&1
  echo "ncu $1 $2 rc=$?"
done
timeout 900 ncu --set full --import-source on --clock-control none -k regex:k_advance -s 2 -c 1 -o $O/adv_C2_bfs python tools/profile_run.py --config C2 --alg bfs --runs 1 > /dev/null 2>&1
timeout 900 ncu --set full --import-source on --clock-control none -k regex:k_filter -s 2 -c 1 -o $O/filt_C2_bfs python tools/profile_run.py --config C2 --alg bfs --runs 1 > /dev/null 2>&1
timeout 900 ncu --set full --import-source on --clock-control none -k regex:k_advance -s 10 -c 1 -o $O/adv_C5_pr python tools/profile_run.py --config C5 --alg pr --runs 1 > /dev/null 2>&1
echo "ncu full rc=$?"
timeout 600 python tools/ablation.py --fsteal --scale 22 --workers 8 --out $O/abl_fsteal_virtual.json
timeout 600 python tools/ablation.py --fsteal --scale 22 --workers 8 --split --out $O/abl_fsteal_split.json
timeout 900 python tools/ablation.py --osteal --grid 2048 --workers 8 --delta 1024 --out $O/abl_osteal_virtual.json
echo done
