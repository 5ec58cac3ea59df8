#!/bin/bash
# filter balance experiment: CTAs per SM x tile swizzle, C2 BFS, seg and degree layouts
O=gpurun_out/r4; mkdir -p $O
for p in seg degree; do
  for n in 0 8 16 32; do for sw in 0 1; do
    if [ $n = 0 ]; then unset GUM_FILTER_CTAS_PER_SM; else export GUM_FILTER_CTAS_PER_SM=$n; fi
    GUM_FILTER_SWIZZLE=$sw python tools/profile_run.py --config C2 --alg bfs --runs 3 --part $p > $O/prof_${p}_n${n}_sw${sw}.txt 2>&1
    echo "$p n=$n sw=$sw $(tail -1 $O/prof_${p}_n${n}_sw${sw}.txt | cut -c1-120)"
  done; done
done
unset GUM_FILTER_CTAS_PER_SM
timeout 300 python bench.py --part degree --no-e2e --no-cpu > $O/bench_C2_degree.json 2> $O/bench_C2_degree.err; echo "bench rc=$?"; tail -c 400 $O/bench_C2_degree.json
