#!/bin/bash
# A/B of filter variants (build/variants/*.so) on C2 BFS (degree layout) and C4 WCC, then the GPU tests and the C2 bench line
O=gpurun_out/fused2; mkdir -p $O
L=build/variants/libgum_new.so,build/variants/libgum_new2.so,build/variants/libgum_new.so,build/variants/libgum_new2.so
timeout 600 python tools/kbench.py --config C2 --alg bfs --part degree --runs 16 --libs $L > $O/kb_c2.txt 2>&1; cat $O/kb_c2.txt
timeout 600 python tools/kbench.py --config C4 --alg wcc --runs 4 --libs build/variants/libgum_new.so,build/variants/libgum_new2.so > $O/kb_c4.txt 2>&1; cat $O/kb_c4.txt
timeout 900 python -m pytest tests -m gpu -q -x > $O/pytest.log 2>&1; echo "pytest rc=$?"; tail -3 $O/pytest.log
timeout 400 python bench.py > $O/bench_C2.json 2> $O/bench_C2.err; echo "C2 rc=$?"; python -c "import json; d=json.loads(open('$O/bench_C2.json').read().strip().splitlines()[-1]); print(d['value'], d['ms_per_step'], d['roofline']['frac'], d['detail']['parity_full_size'])"
