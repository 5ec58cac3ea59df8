O=gpurun_out/ab28; mkdir -p $O
V=build/variants
timeout 900 python tools/kbench.py --config C2 --alg bfs --part degree --runs 10 --libs $V/libgum_fpf0.so,$V/libgum_fpf1.so,$V/libgum_fpf0.so,$V/libgum_fpf1.so > $O/fpf_C2.txt 2>&1; cut -c1-230 $O/fpf_C2.txt
timeout 900 python tools/kbench.py --config C4 --alg wcc --part seg --runs 3 --kw '{"tail_vertices":16384}' --libs $V/libgum_fpf0.so,$V/libgum_fpf1.so > $O/fpf_C4.txt 2>&1; cut -c1-230 $O/fpf_C4.txt
