#!/bin/bash
# full GPU suite, C2 bench (degree layout default), C4 WCC with/without masked blocked dense iterations
O=gpurun_out/r5; mkdir -p $O
timeout 1500 python -m pytest tests -m gpu -q > $O/pytest.log 2>&1; echo "pytest rc=$?"; tail -3 $O/pytest.log
timeout 400 python bench.py > $O/bench_C2.json 2> $O/bench_C2.err; echo "C2 rc=$?"; tail -c 300 $O/bench_C2.json
timeout 900 python bench.py --config C4 --steps 5 --warmup 3 --no-e2e > $O/bench_C4.json 2> $O/bench_C4.err; echo "C4 rc=$?"; tail -c 300 $O/bench_C4.json
GUM_WCC_BLOCKED=0 timeout 900 python bench.py --config C4 --steps 5 --warmup 3 --no-e2e --no-cpu > $O/bench_C4_noblk.json 2> $O/bench_C4_noblk.err; echo "C4 noblk rc=$?"
timeout 900 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none -k regex:k_advance --csv --log-file $O/traffic_C4_wcc.csv python tools/profile_run.py --config C4 --alg wcc --runs 1 > /dev/null 2>&1; echo "ncu C4 rc=$?"
