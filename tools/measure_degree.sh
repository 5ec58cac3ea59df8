mkdir -p gpurun_out/d1
for p in seg degree; do python tools/profile_run.py --config C2 --alg bfs --runs 3 --part $p > gpurun_out/d1/prof_$p.txt 2>&1; done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/d1/launches_C2_bfs_degree.csv python tools/profile_run.py --config C2 --alg bfs --runs 1 --part degree > /dev/null 2>&1
timeout 600 ncu --set full --import-source on --clock-control none -k regex:k_advance -s 2 -c 1 -o gpurun_out/d1/adv_C2_bfs_degree python tools/profile_run.py --config C2 --alg bfs --runs 1 --part degree > /dev/null 2>&1
echo done
