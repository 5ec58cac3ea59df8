O=gpurun_out/ab26; mkdir -p $O
for i in 1 2; do for wo in 0 1024; do
GUM_BFS_WARP_OR_DEG=$wo timeout 600 python tools/kbench.py --config C2 --alg bfs --part degree --runs 10 > $O/wo${wo}_C2_$i.txt 2>&1; echo "C2 wo=$wo $(cut -c1-200 $O/wo${wo}_C2_$i.txt)"
done; done
GUM_BFS_WARP_OR_DEG=1024 timeout 300 python tools/iter_trace.py --config C2 --alg bfs --part degree --runs 5 > $O/iter_C2.txt 2>&1; cat $O/iter_C2.txt
GUM_BFS_WARP_OR_DEG=1 timeout 1200 python -m pytest tests -m gpu -x -q -k "bfs or parity or large" > $O/pytest.txt 2>&1; echo "pytest(all launches warp-or) rc=$?"; tail -2 $O/pytest.txt
