#!/bin/bash
O=gpurun_out/r28; mkdir -p $O
GUM_LIB=build/variants/libgum_old.so timeout 900 python tools/ablation.py --osteal --grid 2048 --workers 8 --delta 1024 --tail 8192 > $O/old.txt 2>&1; echo old; cat $O/old.txt
for n in 1 2; do GUM_TAIL_CTAS_PER_SM=$n timeout 900 python tools/ablation.py --osteal --grid 2048 --workers 8 --delta 1024 --tail 8192 > $O/new$n.txt 2>&1; echo "new tail ctas $n"; cat $O/new$n.txt; done
