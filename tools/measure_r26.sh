#!/bin/bash
O=gpurun_out/r26; mkdir -p $O
for t in 8192 16384; do timeout 900 python tools/ablation.py --osteal --grid 2048 --workers 8 --delta 1024 --tail $t --out $O/abl_osteal_t$t.json > $O/abl_osteal_t$t.txt 2>&1; echo "tail $t"; cat $O/abl_osteal_t$t.txt; done
