O=gpurun_out/dbg1; mkdir -p $O
timeout 1200 python -m pytest tests -m gpu -q -x -k "tail or near_far or units or grid or sssp" > $O/tail.log 2>&1; echo "tests rc=$?"; tail -2 $O/tail.log; grep -E "^E  " $O/tail.log | head
for L in 0 8 16; do GUM_TAIL_LOCAL=$L timeout 900 python tools/kbench.py --config C3 --alg sssp --runs 3 --kw '{"sssp_delta": 4096}' > $O/c3_local$L.txt 2>&1; echo "local=$L"; cat $O/c3_local$L.txt | cut -c1-300; done
