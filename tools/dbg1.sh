O=gpurun_out/dbg1; mkdir -p $O
timeout 1200 python -m pytest tests -m gpu -q -x -k "near_far or tail or sssp or planned or osteal or units" > $O/t.log 2>&1; echo "tests rc=$?"; tail -2 $O/t.log | head -1; grep -E "^E  |FAILED" $O/t.log | head -5
timeout 900 python tools/kbench.py --config C2 --alg bfs --runs 16 --part degree --kw '{"tail_vertices": 0}' --libs build/variants/libgum_db0.so,build/variants/libgum_db1.so,build/variants/libgum_db0.so,build/variants/libgum_db1.so > $O/kb_db.txt 2>&1; cut -c1-260 $O/kb_db.txt
for FL in 0 1; do GUM_FAR_LIST=$FL timeout 900 python tools/kbench.py --config C3 --alg sssp --runs 3 --kw '{"sssp_delta": 4096}' > $O/kb_c3_fl$FL.txt 2>&1; echo "farlist=$FL"; cut -c1-300 $O/kb_c3_fl$FL.txt; done
timeout 900 python tools/ablation.py --table4 --scale 22 --grid 2048 --workers 8 --delta 1024 --out $O/abl_table4.json > $O/abl_table4.txt 2>&1; cat $O/abl_table4.txt
