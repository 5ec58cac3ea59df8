O=gpurun_out/ab17; mkdir -p $O
for tv in 32768 65536 131072; do
timeout 900 python tools/kbench.py --config C3 --alg sssp --part seg --runs 2 --kw "{\"tail_vertices\":$tv,\"sssp_delta\":4096}" > $O/C3_tv${tv}.txt 2>&1; echo "C3 tv=$tv $(cut -c1-200 $O/C3_tv${tv}.txt)"
done
timeout 900 python tools/kbench.py --config C4 --alg wcc --part seg --runs 3 --kw '{"tail_vertices":16384}' > $O/C4.txt 2>&1; echo "C4 $(cut -c1-200 $O/C4.txt)"
