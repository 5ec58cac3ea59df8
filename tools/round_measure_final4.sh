#!/bin/bash
# ncu --set full of the C2 peak-frontier filter (5th launch), filter CTA-count sweep
O=gpurun_out/final4; mkdir -p $O
P="python tools/profile_run.py --runs 1"
timeout 900 ncu --set full --import-source on --clock-control none -k regex:k_filter -s 4 -c 1 -o $O/filt_C2_bfs_peak $P --config C2 --alg bfs --part degree > /dev/null 2>&1
echo "ncu rc=$?"
for n in 4 2 3 4; do echo "filter CTAs/SM=$n"; GUM_FILTER_CTAS_PER_SM=$n timeout 600 python tools/kbench.py --config C2 --alg bfs --part degree --runs 16; done > $O/filter_ctas.txt 2>&1
cat $O/filter_ctas.txt
