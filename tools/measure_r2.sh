#!/bin/bash
# GPU test suite + C2/C4/C5 bench lines under the seg and degree layouts
O=gpurun_out/r2; mkdir -p $O
timeout 1500 python -m pytest tests -m gpu -q > $O/pytest.log 2>&1; echo "pytest rc=$?"; tail -3 $O/pytest.log
for p in seg degree; do
  timeout 300 python bench.py --part $p > $O/bench_C2_$p.json 2> $O/bench_C2_$p.err; echo "C2 $p rc=$?"
  python tools/profile_run.py --config C2 --alg bfs --runs 3 --part $p > $O/prof_C2_$p.txt 2>&1
done
timeout 900 python bench.py --config C4 --steps 5 --warmup 3 --no-e2e --part degree > $O/bench_C4_degree.json 2> $O/bench_C4_degree.err; echo "C4 rc=$?"
timeout 900 python bench.py --config C5 --steps 3 --warmup 3 --no-e2e --part degree > $O/bench_C5_degree.json 2> $O/bench_C5_degree.err; echo "C5 rc=$?"
