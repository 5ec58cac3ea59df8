#!/bin/bash
# round measurement refresh: bench lines C1-C5 (+reference arm), launch lists, ncu of the C2 (degree layout)
# advance and filter, advance DRAM traffic, NEXT-1 traffic ablation
O=gpurun_out/r6; mkdir -p $O
timeout 400 python bench.py > $O/bench_C2.json 2> $O/bench_C2.err; echo "C2 rc=$?"
timeout 300 python bench.py --config C1 --steps 50 > $O/bench_C1.json 2> $O/bench_C1.err; echo "C1 rc=$?"
timeout 900 python bench.py --config C4 --steps 5 --warmup 3 --no-e2e > $O/bench_C4.json 2> $O/bench_C4.err; echo "C4 rc=$?"
timeout 900 python bench.py --config C5 --steps 3 --warmup 3 --no-e2e > $O/bench_C5.json 2> $O/bench_C5.err; echo "C5 rc=$?"
timeout 900 python bench.py --config C3 --steps 3 --warmup 3 --no-e2e > $O/bench_C3.json 2> $O/bench_C3.err; echo "C3 rc=$?"
timeout 600 python bench.py --impl reference --steps 3 > $O/bench_ref_C2.json 2> $O/bench_ref_C2.err; echo "ref rc=$?"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_C2_bfs.csv python tools/profile_run.py --config C2 --alg bfs --runs 1 --part degree > /dev/null 2>&1
timeout 900 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none -k regex:k_advance --csv --log-file $O/traffic_C2_bfs.csv python tools/profile_run.py --config C2 --alg bfs --runs 1 --part degree > /dev/null 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_C4_wcc.csv python tools/profile_run.py --config C4 --alg wcc --runs 1 > /dev/null 2>&1
timeout 900 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none -k regex:k_advance --csv --log-file $O/traffic_C4_wcc.csv python tools/profile_run.py --config C4 --alg wcc --runs 1 > /dev/null 2>&1
echo "ncu lists done"
timeout 900 ncu --set full --import-source on --clock-control none -k regex:k_advance -s 2 -c 1 -o $O/adv_C2_bfs python tools/profile_run.py --config C2 --alg bfs --runs 1 --part degree > /dev/null 2>&1
timeout 900 ncu --set full --import-source on --clock-control none -k regex:k_filter -s 2 -c 1 -o $O/filt_C2_bfs python tools/profile_run.py --config C2 --alg bfs --runs 1 --part degree > /dev/null 2>&1
echo "ncu full done"
timeout 900 python tools/ablation.py --next1 --scale 20 --workers 8 --out $O/abl_next1.json > $O/abl_next1.txt 2>&1; echo "next1 rc=$?"
echo done
