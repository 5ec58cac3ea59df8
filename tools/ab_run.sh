O=gpurun_out/ab4; mkdir -p $O
( time timeout 1200 python -m pytest tests -m gpu -x -q ) > $O/pytest.txt 2>&1; echo "pytest rc=$?"; tail -4 $O/pytest.txt
for i in 1 2; do for vf in 0 1; do
GUM_BFS_VIS_FILTER=$vf timeout 600 python tools/kbench.py --config C2 --alg bfs --part degree --runs 10 > $O/vf${vf}_C2_$i.txt 2>&1; echo "C2 vf=$vf $(cat $O/vf${vf}_C2_$i.txt)"
done; done
for vf in 0 1; do
GUM_BFS_VIS_FILTER=$vf timeout 600 python tools/kbench.py --config C1 --alg bfs --part degree --runs 20 > $O/vf${vf}_C1.txt 2>&1; echo "C1 vf=$vf $(cat $O/vf${vf}_C1.txt)"
done
timeout 300 python tools/iter_trace.py --config C2 --alg bfs --part degree --runs 5 > $O/iter_C2.txt 2>&1; cat $O/iter_C2.txt
