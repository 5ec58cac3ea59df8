O=gpurun_out/ab16; mkdir -p $O
GUM_TAIL_SLACK=0 timeout 600 python -c "
import sys; sys.path.insert(0, '.')
import tests.test_gpu_tail_nodedupe as t
exec(t.CHILD.replace('ROOT', repr('.')))
" > $O/ovf.txt 2>&1; echo "ovf rc=$?"; tail -2 $O/ovf.txt
for tl in 8 16 32; do for tv in 16384 32768; do
GUM_TAIL_LOCAL=$tl timeout 900 python tools/kbench.py --config C3 --alg sssp --part seg --runs 2 --kw "{\"tail_vertices\":$tv,\"sssp_delta\":4096}" > $O/C3_tl${tl}_tv${tv}.txt 2>&1; echo "C3 tl=$tl tv=$tv $(cut -c1-220 $O/C3_tl${tl}_tv${tv}.txt)"
done; done
for d in 2048 8192; do
timeout 900 python tools/kbench.py --config C3 --alg sssp --part seg --runs 2 --kw "{\"tail_vertices\":16384,\"sssp_delta\":$d}" > $O/C3_d$d.txt 2>&1; echo "C3 delta=$d $(cut -c1-220 $O/C3_d$d.txt)"
done
bash tools/ncu_longest.sh $O/ncu k_tail --config C3 --alg sssp --runs 1
