O=gpurun_out/ab24; mkdir -p $O
for i in 1 2; do for hd in 0 1; do
GUM_BFS_HOT_DD=$hd timeout 600 python tools/kbench.py --config C2 --alg bfs --part degree --runs 10 > $O/hd${hd}_C2_$i.txt 2>&1; echo "C2 hd=$hd $(cut -c1-200 $O/hd${hd}_C2_$i.txt)"
done; done
for hd in 0 1; do GUM_BFS_HOT_DD=$hd timeout 600 python tools/kbench.py --config C1 --alg bfs --part degree --runs 30 > $O/hd${hd}_C1.txt 2>&1; echo "C1 hd=$hd $(cut -c1-200 $O/hd${hd}_C1.txt)"; done
timeout 300 python tools/iter_trace.py --config C2 --alg bfs --part degree --runs 5 > $O/iter_C2.txt 2>&1; cat $O/iter_C2.txt
timeout 1200 python -m pytest tests -m gpu -x -q -k "bfs or parity or large or filter" > $O/pytest.txt 2>&1; echo "pytest rc=$?"; tail -2 $O/pytest.txt
