#!/bin/bash
O=gpurun_out/r20; mkdir -p $O
for n in 2 3; do GUM_TAIL_CTAS_PER_SM=$n timeout 900 python tools/ablation.py --osteal --grid 2048 --workers 8 --delta 1024 > $O/abl_osteal_$n.txt 2>&1; echo "tail ctas $n"; cat $O/abl_osteal_$n.txt; done
for v in fminb3 fminb2; do GUM_LIB=build/variants/libgum_$v.so python tools/profile_run.py --config C2 --alg bfs --runs 3 --part degree > $O/prof_$v.txt 2>&1; echo "$v $(tail -1 $O/prof_$v.txt | cut -c1-120)"; done
python tools/profile_run.py --config C2 --alg bfs --runs 3 --part degree > $O/prof_base.txt 2>&1; echo "base $(tail -1 $O/prof_base.txt | cut -c1-120)"
